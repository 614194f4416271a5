// internal.h — host-side internals of libcst (not part of the C ABI).
#pragma once

#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <array>
#include <cstdint>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "../../../include/cst.h"
#include "../kernels/cst_params.h"

namespace cst {

// ------------------------------------------------------------------ error handling
void set_error(const std::string& msg);
cst_status fail(cst_status s, const std::string& msg);
#define CST_CUDA(call)                                                              \
  do {                                                                              \
    cudaError_t e_ = (call);                                                        \
    if (e_ != cudaSuccess)                                                          \
      return ::cst::fail(CST_E_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

// ------------------------------------------------------------------ settings
// The 21 fields in canonical order: Table I row order, then the temporal
// blocking degree (B200 extension, NEXT-2) and the streamed-state store (qstore, TMEM).
enum Field {
  F_TBX, F_TBY, F_TBZ, F_STAGING, F_CONST, F_STREAM, F_SD, F_SB, F_UFX, F_UFY, F_UFZ,
  F_CMX, F_CMY, F_CMZ, F_BMX, F_BMY, F_BMZ, F_RET, F_PF, F_BT, F_QS, F_COUNT
};
using Tuple = std::array<int32_t, F_COUNT>;
Tuple to_tuple(const cst_setting& s);
cst_setting from_tuple(const Tuple& t);
std::string setting_key(const cst_setting& s);
extern const char* const kFieldNames[F_COUNT];

struct StencilInfo {
  int kind, r;
  int64_t M[3];  // nx, ny, nz
};

// Rule check (R1..R12, R14, R15).  Returns nullptr if valid else the rule id.
const char* check_rules(const StencilInfo& st, const Tuple& t);
int64_t model_smem_bytes(int kind, int r, const Tuple& t);
int64_t model_regs(int kind, int r, const Tuple& t);
int64_t uf_trip(int kind, const Tuple& t, int d);
// R16: the setting selects rhs4's retimed column-walk kernel (kernel_rhs4_ret)
bool r4ret_path(int kind, const Tuple& t);
// TMEM columns one CTA of the qstore = 2 path allocates (power of two >= 32)
int tmem_cols_alloc(int kind, int r, const Tuple& t);
// Dynamic shared memory the kernel variant actually uses (<= model for fast paths).
int64_t kernel_smem_bytes(int kind, int r, const Tuple& t);
bool hyp_trimmed(int kind, const Tuple& t);
void stream_array_box(int kind, int r, const Tuple& t, int a, int64_t* wa, int64_t* wb);

// ------------------------------------------------------------------ space
class Space {
 public:
  explicit Space(const StencilInfo& st);
  uint64_t count() const { return total_; }
  bool at(uint64_t rank, Tuple* out) const;
  bool rank(const Tuple& t, uint64_t* out) const;
  // Stream the valid settings of prefixes [p0, p1) in rank order: f(rank, tuple).  The
  // prefixes (first 8 fields) partition the space, so threads can split them.
  size_t n_prefixes() const { return prefixes_.size(); }
  uint64_t prefix_start(size_t i) const { return prefixes_[i].start; }
  template <class F>
  void for_each(size_t p0, size_t p1, F&& f) const;

 private:
  struct Core {  // (CM x3, BM x3, ret, pf, bt, qs) and its per-dim UF bounds (counts)
    int32_t cm[3], bm[3], ret, pf, bt, qs;
    int32_t nuf[3];
  };
  struct Prefix {
    int32_t v[8];       // TBx TBy TBz staging const streaming SD SB
    uint64_t start;     // cumulative rank of the first completion
    uint64_t count;
  };
  void cores_for(const int32_t* prefix, std::vector<Core>* cores) const;
  StencilInfo st_;
  uint64_t id_;                 // unique per Space (keys at()'s per-thread core cache)
  std::vector<Prefix> prefixes_;
  uint64_t total_ = 0;
  std::vector<int32_t> p2_[3];  // powers of two <= M_d
};

template <class F>
void Space::for_each(size_t p0, size_t p1, F&& f) const {
  std::vector<Core> cores;
  for (size_t pi = p0; pi < p1 && pi < prefixes_.size(); ++pi) {
    const Prefix& P = prefixes_[pi];
    cores_for(P.v, &cores);
    Tuple t{};
    for (int i = 0; i < 8; ++i) t[i] = P.v[i];
    uint64_t rk = P.start;
    // canonical order within a prefix: UF_x, UF_y, UF_z, then the cores (see Space::at)
    for (int32_t u0 = 0; u0 < (int32_t)p2_[0].size(); ++u0)
      for (int32_t u1 = 0; u1 < (int32_t)p2_[1].size(); ++u1)
        for (int32_t u2 = 0; u2 < (int32_t)p2_[2].size(); ++u2)
          for (const Core& c : cores) {
            if (u0 >= c.nuf[0] || u1 >= c.nuf[1] || u2 >= c.nuf[2]) continue;
            t[F_UFX] = p2_[0][u0];
            t[F_UFY] = p2_[1][u1];
            t[F_UFZ] = p2_[2][u2];
            for (int d = 0; d < 3; ++d) {
              t[F_CMX + d] = c.cm[d];
              t[F_BMX + d] = c.bm[d];
            }
            t[F_RET] = c.ret;
            t[F_PF] = c.pf;
            t[F_BT] = c.bt;
            t[F_QS] = c.qs;
            f(rk++, t);
          }
  }
}

// Copy the logical halo of one array (fill.cu).  Multi-step sweeps use in[]'s halo as the
// boundary condition of every step.
// zlo / zhi: include the z-halo planes below / above whole (false where a z-slab neighbour
// fills their interior x/y: then only their x/y ring is copied).
cst_status copy_halo(const cst_grid& g, const double* src, double* dst, cudaStream_t stream,
                     bool zlo = true, bool zhi = true);

// Peer-memory halo transport (dist/p2p.cu): signal = after the stream's prior work, store
// `value` (release, system scope) into every non-null flag word; wait = block the stream
// until every non-null flag word >= its target (acquire, 30 s bound, then trap).
cst_status p2p_signal(cudaStream_t s, unsigned long long* f0, unsigned long long* f1,
                      unsigned long long value);
cst_status p2p_wait(cudaStream_t s, const unsigned long long* f0, unsigned long long t0,
                    const unsigned long long* f1, unsigned long long t1);

// Temporal-blocking pass schedule: step counts per kernel pass (powers of two <= bt)
// summing to nsteps, with as many passes as nsteps has parity (ping-pong placement).
std::vector<int> pass_schedule(int nsteps, int bt);

// ------------------------------------------------------------------ driver entry points
struct Driver {
  PFN_cuModuleLoadData_v2000 cuModuleLoadData = nullptr;
  PFN_cuModuleUnload_v2000 cuModuleUnload = nullptr;
  PFN_cuModuleGetFunction_v2000 cuModuleGetFunction = nullptr;
  PFN_cuModuleGetGlobal_v3020 cuModuleGetGlobal = nullptr;
  PFN_cuFuncSetAttribute_v9000 cuFuncSetAttribute = nullptr;
  PFN_cuFuncGetAttribute_v2020 cuFuncGetAttribute = nullptr;
  PFN_cuLaunchKernel_v4000 cuLaunchKernel = nullptr;
  PFN_cuTensorMapEncodeTiled_v12000 cuTensorMapEncodeTiled = nullptr;
  PFN_cuOccupancyMaxActiveBlocksPerMultiprocessor_v6050 cuOccupancy = nullptr;
  PFN_cuGetErrorString_v6000 cuGetErrorString = nullptr;
  PFN_cuMemGetAddressRange_v3020 cuMemGetAddressRange = nullptr;
};
cst_status driver(const Driver** out);
cst_status cu_check(CUresult r, const char* what);

// ------------------------------------------------------------------ JIT
struct Variant {
  CUmodule mod = nullptr;
  CUfunction fn = nullptr;
  int smem = 0;
  int regs = 0;
  int local = 0;
  int threads = 0;
  int occ = 0;
  double compile_s = 0;
  bool coef_uploaded = false;
};
// Compile (or fetch from the memory/disk cache) the cubin of a variant; remote = the
// fused-halo twin whose stores also go to the neighbour's halo (CST_REMOTE).
cst_status jit_cubin(const StencilInfo& st, const Tuple& t, std::string* cubin,
                     double* compile_s,
                     bool remote = false);
uint64_t jit_compile_count();
std::string nvrtc_description();

}  // namespace cst

// Launch one sweep of local interior planes [z0, z0 + nz) (sub-domain sweeps).  rout
// (optional, one per output): every stored value also goes to rout[q] + (element offset
// of the point relative to element (0, 0, z0) of out[q]) — the fused halo exchange.
cst_status cst_launch_range(cst_stencil* h, const cst_setting* s, const double* const* in,
                            double* const* out, int64_t z0, int64_t nz, cudaStream_t stream,
                            double* const* rout = nullptr);
// Resolve (compile, load, check R13) the variant of a setting — and its fused-halo twin if
// `remote` — without launching anything (so multi-rank protocols fail before they start).
cst_status cst_resolve_variant(cst_stencil* h, const cst_setting* s, bool remote);

namespace cst {

}  // namespace cst

struct cst_stencil {
  cst_stencil_desc desc{};
  std::vector<double> coeffs;   // as given (desc.n_coeffs)
  std::vector<double> kcoef;    // kernel coefficient bank (coeffs + derived weights)
  cst_grid grid{};
  int device = 0;
  int num_sms = 0;              // SMs of the device (persistent launches); 0 = unknown
  cst::StencilInfo info{};
  std::unique_ptr<cst::Space> space;
  std::map<std::string, cst::Variant> variants;
  // TMA descriptor cache: (array base pointer, box dims) -> map
  std::map<std::array<int64_t, 4>, cst_tmap> tmaps;
  // host-path staging
  std::vector<double*> dev_bufs;
  size_t dev_buf_elems = 0;
  cudaStream_t host_stream = nullptr;
  cudaStream_t host_in_stream = nullptr, host_out_stream = nullptr;
  int64_t last_launches = 0;
};
