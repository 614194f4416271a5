// cst_api.cpp — C ABI of libcst (include/cst.h): handles, validation, space queries,
// variant loading (JIT modules, TMA descriptors), sweeps and timing.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstring>
#include <cstdlib>
#include <mutex>

#include "internal.h"

namespace cst {

static thread_local std::string t_err;

void set_error(const std::string& msg) { t_err = msg; }

cst_status fail(cst_status s, const std::string& msg) {
  t_err = msg;
  return s;
}

cst_status cu_check(CUresult r, const char* what) {
  if (r == CUDA_SUCCESS) return CST_OK;
  const Driver* d = nullptr;
  const char* s = nullptr;
  if (driver(&d) == CST_OK && d->cuGetErrorString) d->cuGetErrorString(r, &s);
  return fail(CST_E_CUDA, std::string(what) + ": CUresult " + std::to_string((int)r) + " " +
                              (s ? s : ""));
}

cst_status driver(const Driver** out) {
  static Driver d;
  static cst_status st = CST_E_INTERNAL;
  static std::string err;
  static std::once_flag once;
  std::call_once(once, [] {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
      cudaGetLastError();
      st = CST_E_CUDA;
      err = "no CUDA device available (libcst has no CPU fallback)";
      return;
    }
    auto get = [](const char* name, void** fp) {
      cudaDriverEntryPointQueryResult q;
      return cudaGetDriverEntryPoint(name, fp, cudaEnableDefault, &q) == cudaSuccess &&
             q == cudaDriverEntryPointSuccess && *fp;
    };
    bool ok = get("cuModuleLoadData", (void**)&d.cuModuleLoadData) &&
              get("cuModuleUnload", (void**)&d.cuModuleUnload) &&
              get("cuModuleGetFunction", (void**)&d.cuModuleGetFunction) &&
              get("cuModuleGetGlobal", (void**)&d.cuModuleGetGlobal) &&
              get("cuFuncSetAttribute", (void**)&d.cuFuncSetAttribute) &&
              get("cuFuncGetAttribute", (void**)&d.cuFuncGetAttribute) &&
              get("cuLaunchKernel", (void**)&d.cuLaunchKernel) &&
              get("cuTensorMapEncodeTiled", (void**)&d.cuTensorMapEncodeTiled) &&
              get("cuOccupancyMaxActiveBlocksPerMultiprocessor", (void**)&d.cuOccupancy) &&
              get("cuGetErrorString", (void**)&d.cuGetErrorString) &&
              get("cuMemGetAddressRange", (void**)&d.cuMemGetAddressRange);
    if (!ok) {
      st = CST_E_CUDA;
      err = "cudaGetDriverEntryPoint failed for a required driver function";
      return;
    }
    st = CST_OK;
  });
  if (st != CST_OK) return fail(st, err);
  *out = &d;
  return CST_OK;
}

// ------------------------------------------------------------------ launch geometry
struct Geometry {
  unsigned grid_x, grid_y, threads;
  int tiles_a, tiles_b, tiles_c, chunks;
  int box[3];  // TMA box dims (x, y, z)
};

static int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

static Geometry geometry(const StencilInfo& st, const Tuple& t, int64_t nx, int64_t ny,
                         int64_t nz) {
  Geometry g{};
  const int r = st.r;
  const int xr = r + (r & 1);  // even x halo of the smem/TMA boxes (kernels' XR)
  int64_t T[3];
  for (int d = 0; d < 3; ++d) T[d] = (int64_t)t[F_TBX + d] * t[F_BMX + d] * t[F_CMX + d];
  g.threads = (unsigned)(t[F_TBX] * t[F_TBY] * t[F_TBZ]);
  if (t[F_STREAM] == 2) {
    const bool sz = t[F_SD] == 3;
    g.tiles_a = (int)cdiv(nx, T[0]);
    g.tiles_b = (int)cdiv(sz ? ny : nz, sz ? T[1] : T[2]);
    g.chunks = (int)cdiv(sz ? nz : ny, t[F_SB]);
    g.tiles_c = 1;
    g.grid_x = (unsigned)(g.tiles_a * (int64_t)g.tiles_b);
    g.grid_y = (unsigned)g.chunks;
    g.box[0] = (int)T[0] + 2 * xr;
    if (t[F_BT] > 1) {  // temporally blocked: the input box carries bt halos per side
      g.box[0] = (int)T[0] + 2 * xr * t[F_BT];
      g.box[1] = (int)T[1] + 2 * r * t[F_BT];
      g.box[2] = 1;
    } else if (sz) {
      g.box[1] = (int)T[1] + 2 * r;
      g.box[2] = 1;
    } else {
      g.box[1] = 1;
      g.box[2] = (int)T[2] + 2 * r;
    }
  } else {
    g.tiles_a = (int)cdiv(nx, T[0]);
    g.tiles_b = (int)cdiv(ny, T[1]);
    g.tiles_c = (int)cdiv(nz, T[2]);
    g.chunks = 1;
    g.grid_x = (unsigned)(g.tiles_a * (int64_t)g.tiles_b);
    g.grid_y = (unsigned)g.tiles_c;
    for (int d = 0; d < 3; ++d) g.box[d] = (int)T[d] + 2 * (d == 0 ? xr : r);
  }
  return g;
}

}  // namespace cst

using namespace cst;

// ====================================================================== status
extern "C" const char* cst_status_str(cst_status s) {
  switch (s) {
    case CST_OK: return "CST_OK";
    case CST_E_INVALID: return "CST_E_INVALID";
    case CST_E_UNSUPPORTED: return "CST_E_UNSUPPORTED";
    case CST_E_CONSTRAINT: return "CST_E_CONSTRAINT";
    case CST_E_CUDA: return "CST_E_CUDA";
    case CST_E_NVRTC: return "CST_E_NVRTC";
    case CST_E_NCCL: return "CST_E_NCCL";
    case CST_E_OOM: return "CST_E_OOM";
    case CST_E_INTERNAL: return "CST_E_INTERNAL";
  }
  return "CST_E_?";
}

extern "C" const char* cst_last_error(void) { return t_err.c_str(); }
extern "C" const char* cst_version(void) {
  static std::string v = "cst 0.1 (sm_100a; " + nvrtc_description() + ")";
  return v.c_str();
}

// ====================================================================== handles
static int expected_coeffs(int kind, int r) {
  if (kind == CST_STAR) return 6 * r + 1;
  if (kind == CST_BOX) return (2 * r + 1) * (2 * r + 1) * (2 * r + 1);
  if (kind == CST_RHS4) return 3;
  return 7;
}

extern "C" cst_status cst_stencil_create(const cst_stencil_desc* desc, const cst_grid* g,
                                         int device, cst_stencil** out) {
  if (!desc || !g || !out) return fail(CST_E_INVALID, "null argument");
  const int kind = desc->kind, r = desc->order;
  const bool supported = (kind == CST_STAR && r >= 1 && r <= 4) ||
                         (kind == CST_BOX && r == 1) || (kind == CST_HYPTERM && r == 4) ||
                         (kind == CST_RHS4 && r == 2);
  if (kind < 1 || kind > 4) return fail(CST_E_INVALID, "desc.kind");
  if (!supported) return fail(CST_E_UNSUPPORTED, "(kind, order) not supported");
  const int nin = kind == CST_HYPTERM ? 8 : (kind == CST_RHS4 ? 5 : 1);
  const int nout = kind == CST_HYPTERM ? 5 : (kind == CST_RHS4 ? 3 : 1);
  if (desc->n_inputs != nin || desc->n_outputs != nout)
    return fail(CST_E_INVALID, "desc.n_inputs / n_outputs do not match the kind");
  if (!desc->coeffs || desc->n_coeffs != expected_coeffs(kind, r))
    return fail(CST_E_INVALID, "desc.coeffs / n_coeffs (expected " +
                                   std::to_string(expected_coeffs(kind, r)) + ")");
  for (int i = 0; i < desc->n_coeffs; ++i)
    if (!std::isfinite(desc->coeffs[i])) return fail(CST_E_INVALID, "non-finite coefficient");
  if (g->nx < 1 || g->ny < 1 || g->nz < 1) return fail(CST_E_INVALID, "grid extents < 1");
  if (g->nx > (1 << 30) || g->ny > (1 << 30) || g->nz > (1 << 30))
    return fail(CST_E_UNSUPPORTED, "grid extent too large");
  if (g->halo < r) return fail(CST_E_INVALID, "grid.halo < order");
  if (g->lead_x < g->halo) return fail(CST_E_INVALID, "grid.lead_x < halo");
  if (g->pitch_x < g->lead_x + g->nx + g->halo || (g->pitch_x % 2))
    return fail(CST_E_INVALID, "grid.pitch_x must be even and >= lead_x + nx + halo");
  if (g->pitch_y < g->ny + 2 * g->halo) return fail(CST_E_INVALID, "grid.pitch_y < ny + 2*halo");
  if (device < 0) return fail(CST_E_INVALID, "device < 0");
  auto* h = new cst_stencil();
  h->desc = *desc;
  h->coeffs.assign(desc->coeffs, desc->coeffs + desc->n_coeffs);
  h->desc.coeffs = h->coeffs.data();
  // kernel coefficient bank: the user's coefficients, plus for hypterm the derivative
  // weight magnitudes P_d[j] = dxinv_d a_j (j = 1..4) for d = z, y, x — the kernels apply
  // w_d[k] = -sign(k) P_d[|k|] (streamed direction and row-streamed in-plane terms)
  h->kcoef = h->coeffs;
  if (kind == CST_RHS4) {
    // s_d^2 / 6 for the V terms, s_d s_i / 144 for the mixed pairs (0,1), (0,2), (1,2)
    for (int d = 0; d < 3; ++d) h->kcoef.push_back(h->coeffs[d] * h->coeffs[d] / 6.0);
    h->kcoef.push_back(h->coeffs[0] * h->coeffs[1] / 144.0);
    h->kcoef.push_back(h->coeffs[0] * h->coeffs[2] / 144.0);
    h->kcoef.push_back(h->coeffs[1] * h->coeffs[2] / 144.0);
  }
  if (kind == CST_HYPTERM)
    for (int sdir : {2, 1, 0})
      for (int j = 1; j <= 4; ++j) h->kcoef.push_back(h->coeffs[4 + sdir] * h->coeffs[j - 1]);
  h->grid = *g;
  h->device = device;
  {
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) {
      cudaGetLastError();
      n = 0;
    }
    h->num_sms = n;
  }
  h->info.kind = kind;
  h->info.r = r;
  h->info.M[0] = g->nx;
  h->info.M[1] = g->ny;
  h->info.M[2] = g->nz;
  *out = h;
  return CST_OK;
}

extern "C" void cst_stencil_destroy(cst_stencil* h) {
  if (!h) return;
  const Driver* d = nullptr;
  if (driver(&d) == CST_OK) {
    cudaSetDevice(h->device);
    for (auto& kv : h->variants)
      if (kv.second.mod) d->cuModuleUnload(kv.second.mod);
    for (double* p : h->dev_bufs) cudaFree(p);
    if (h->host_stream) cudaStreamDestroy(h->host_stream);
    if (h->host_in_stream) cudaStreamDestroy(h->host_in_stream);
    if (h->host_out_stream) cudaStreamDestroy(h->host_out_stream);
  }
  delete h;
}

extern "C" cst_status cst_setting_check(const cst_stencil* h, const cst_setting* s) {
  if (!h || !s) return fail(CST_E_INVALID, "null argument");
  const char* rule = check_rules(h->info, to_tuple(*s));
  if (rule) return fail(CST_E_CONSTRAINT, std::string("setting violates ") + rule);
  return CST_OK;
}

extern "C" cst_status cst_setting_default(const cst_stencil* h, cst_setting* s) {
  if (!h || !s) return fail(CST_E_INVALID, "null argument");
  auto p2floor = [](int64_t v, int64_t cap) {
    int64_t x = 1;
    while (x * 2 <= v && x * 2 <= cap) x *= 2;
    return (int32_t)x;
  };
  const int64_t* M = h->info.M;
  // measured-good starting points on B200, shrunk to fit small grids:
  // streaming along z, TMA staging, retimed accumulators; star/box 64x8 tiles of 2x2
  // register blocks; rhs4 the retimed column walk, 8x16 threads with two x-adjacent points
  // each, 64-plane blocks, 1-deep prefetch, coefficients in __constant__ (0.965 vs 1.095 ms
  // for the generic path at 320^3); hypterm 32x4 threads with two points
  // stacked along y each, streamed state in TMEM, x-product planes with a 2-deep ring,
  // coefficients in __constant__.
  const bool hyp = h->info.kind == CST_HYPTERM || h->info.kind == CST_RHS4;
  const bool hyp_tm = h->info.kind == CST_HYPTERM;
  const bool r4 = h->info.kind == CST_RHS4;
  cst_setting c{};
  c.tb[0] = r4 ? 8 : 32;
  c.tb[1] = r4 ? 16 : 4;
  c.tb[2] = 1;
  c.staging = 3;
  c.use_constant = 1;
  c.use_streaming = 2;
  c.sd = 3;
  c.sb = p2floor(M[2], h->info.kind == CST_HYPTERM ? 256 : (r4 ? 64 : 128));
  for (int d = 0; d < 3; ++d) c.uf[d] = c.cm[d] = c.bm[d] = 1;
  c.bm[0] = hyp && !r4 ? 1 : 2;
  c.bm[1] = r4 ? 1 : 2;
  c.use_retiming = 2;
  c.bt = 1;
  c.qstore = hyp_tm ? 2 : 1;
  if (hyp) c.use_constant = 2;
  c.prefetch = (h->info.kind == CST_BOX || hyp_tm) ? 2 : (r4 ? 1 : 3);
  for (int tries = 0; tries < 12 && check_rules(h->info, to_tuple(c)); ++tries) {
    if (c.qstore == 2 && c.staging != 3) { c.qstore = 1; continue; }  // R15 needs TMA
    // shrink the tile until it fits the grid (coverage) and the thread floor
    if (c.bm[0] > 1 && (int64_t)c.tb[0] * c.bm[0] > M[0]) c.bm[0] /= 2;
    else if (c.bm[1] > 1 && (int64_t)c.tb[1] * c.bm[1] > M[1]) c.bm[1] /= 2;
    else if (c.tb[0] > 1 && c.tb[0] > M[0]) { c.tb[0] /= 2; c.tb[1] *= 2; }
    else if (c.tb[1] > 1 && c.tb[1] > M[1]) { c.tb[1] /= 2; }
    else if (c.tb[0] * c.bm[0] % 2) { c.staging = 2; }
    else if (c.qstore == 2) { c.qstore = 1; }
    else if (r4 && c.use_retiming == 2) { c.use_retiming = 1; }  // R16 needs TMA staging
    else break;
  }
  if (!check_rules(h->info, to_tuple(c))) {
    *s = c;
    return CST_OK;
  }
  // fall back to the first valid setting of the canonical space
  cst_stencil* hh = const_cast<cst_stencil*>(h);
  if (!hh->space) hh->space.reset(new Space(h->info));
  Tuple t;
  if (!hh->space->at(0, &t)) return fail(CST_E_CONSTRAINT, "empty parameter space");
  *s = from_tuple(t);
  return CST_OK;
}

// ====================================================================== space
extern "C" cst_status cst_space_count(cst_stencil* h, uint64_t* n) {
  if (!h || !n) return fail(CST_E_INVALID, "null argument");
  if (!h->space) h->space.reset(new Space(h->info));
  *n = h->space->count();
  return CST_OK;
}

extern "C" cst_status cst_space_at(cst_stencil* h, uint64_t rank, cst_setting* s) {
  if (!h || !s) return fail(CST_E_INVALID, "null argument");
  if (!h->space) h->space.reset(new Space(h->info));
  Tuple t;
  if (!h->space->at(rank, &t)) return fail(CST_E_INVALID, "rank out of range");
  *s = from_tuple(t);
  return CST_OK;
}

extern "C" cst_status cst_space_rank(cst_stencil* h, const cst_setting* s, uint64_t* rank) {
  if (!h || !s || !rank) return fail(CST_E_INVALID, "null argument");
  if (!h->space) h->space.reset(new Space(h->info));
  const char* rule = check_rules(h->info, to_tuple(*s));
  if (rule) return fail(CST_E_CONSTRAINT, std::string("setting violates ") + rule);
  uint64_t r;
  if (!h->space->rank(to_tuple(*s), &r)) return fail(CST_E_INTERNAL, "rank lookup failed");
  *rank = r;
  return CST_OK;
}

// ====================================================================== variants
static cst_status get_variant(cst_stencil* h, const cst_setting* s, Variant** out,
                              bool remote = false) {
  const char* rule = check_rules(h->info, to_tuple(*s));
  if (rule) return fail(CST_E_CONSTRAINT, std::string("setting violates ") + rule);
  const std::string key = setting_key(*s) + (remote ? ",remote" : "");
  auto it = h->variants.find(key);
  if (it != h->variants.end()) {
    if (!it->second.fn)
      return fail(CST_E_CONSTRAINT, "R13: variant rejected (" + std::string("spill/smem") + ")");
    *out = &it->second;
    return CST_OK;
  }
  const Driver* d = nullptr;
  cst_status st = driver(&d);
  if (st != CST_OK) return st;
  CST_CUDA(cudaSetDevice(h->device));
  CST_CUDA(cudaFree(nullptr));  // make sure the primary context exists and is current
  const Tuple t = to_tuple(*s);
  const int64_t smem = kernel_smem_bytes(h->info.kind, h->info.r, t);
  Variant v;
  if (smem > 227 * 1024) {
    h->variants[key] = v;  // remember the rejection
    return fail(CST_E_CONSTRAINT, "R10: kernel shared memory " + std::to_string(smem) +
                                      " B exceeds 227 KiB");
  }
  std::string cubin;
  st = jit_cubin(h->info, t, &cubin, &v.compile_s, remote);
  if (st != CST_OK) return st;
  st = cu_check(d->cuModuleLoadData(&v.mod, cubin.data()), "cuModuleLoadData");
  if (st != CST_OK) return st;
  st = cu_check(d->cuModuleGetFunction(&v.fn, v.mod, "cst_kernel"), "cuModuleGetFunction");
  if (st != CST_OK) return st;
  v.smem = (int)smem;
  v.threads = t[F_TBX] * t[F_TBY] * t[F_TBZ];
  d->cuFuncGetAttribute(&v.regs, CU_FUNC_ATTRIBUTE_NUM_REGS, v.fn);
  d->cuFuncGetAttribute(&v.local, CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES, v.fn);
  if (smem > 48 * 1024) {
    st = cu_check(d->cuFuncSetAttribute(v.fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES,
                                        (int)smem),
                  "cuFuncSetAttribute(smem)");
    if (st != CST_OK) return st;
  }
  if (d->cuOccupancy(&v.occ, v.fn, v.threads, (size_t)smem) != CUDA_SUCCESS) v.occ = 0;
  if (v.local > 0 || v.occ == 0) {
    d->cuModuleUnload(v.mod);
    Variant rej;
    rej.compile_s = v.compile_s;
    rej.regs = v.regs;
    rej.local = v.local;
    h->variants[key] = rej;
    return fail(CST_E_CONSTRAINT,
                v.local > 0 ? "R13: variant spills to local memory (" +
                                  std::to_string(v.local) + " B/thread)"
                            : "R13: variant cannot be resident (occupancy 0)");
  }
  if (t[F_CONST] == 2) {
    CUdeviceptr dp;
    size_t bytes;
    st = cu_check(d->cuModuleGetGlobal(&dp, &bytes, v.mod, "c_coef"), "cuModuleGetGlobal");
    if (st != CST_OK) return st;
    CST_CUDA(cudaMemcpy((void*)dp, h->kcoef.data(), h->kcoef.size() * sizeof(double),
                        cudaMemcpyHostToDevice));
  }
  h->variants[key] = v;
  *out = &h->variants[key];
  return CST_OK;
}

cst_status cst_resolve_variant(cst_stencil* h, const cst_setting* s, bool remote) {
  Variant* v = nullptr;
  cst_status st = get_variant(h, s, &v, false);
  if (st == CST_OK && remote) st = get_variant(h, s, &v, true);
  return st;
}

extern "C" cst_status cst_variant_compile(const cst_stencil* h, const cst_setting* s,
                                          double* compile_s) {
  if (!h || !s || !compile_s) return fail(CST_E_INVALID, "null argument");
  const Tuple t = to_tuple(*s);
  const char* rule = check_rules(h->info, t);
  if (rule) return fail(CST_E_CONSTRAINT, std::string("setting violates ") + rule);
  std::string cubin;
  return jit_cubin(h->info, t, &cubin, compile_s);
}

extern "C" cst_status cst_variant_cubin(const cst_stencil* h, const cst_setting* s,
                                        int32_t remote, void* buf, int64_t cap, int64_t* size) {
  if (!h || !s || !size || (cap > 0 && !buf)) return fail(CST_E_INVALID, "null argument");
  const Tuple t = to_tuple(*s);
  const char* rule = check_rules(h->info, t);
  if (rule) return fail(CST_E_CONSTRAINT, std::string("setting violates ") + rule);
  std::string cubin;
  double cs = 0;
  const cst_status st = jit_cubin(h->info, t, &cubin, &cs, remote != 0);
  if (st != CST_OK) return st;
  *size = (int64_t)cubin.size();
  if (cap < (int64_t)cubin.size()) return fail(CST_E_INVALID, "cst_variant_cubin: buffer too small");
  std::memcpy(buf, cubin.data(), cubin.size());
  return CST_OK;
}

extern "C" cst_status cst_kernel_info_get(cst_stencil* h, const cst_setting* s,
                                          cst_kernel_info* info) {
  if (!h || !s || !info) return fail(CST_E_INVALID, "null argument");
  Variant* v = nullptr;
  cst_status st = get_variant(h, s, &v);
  if (st != CST_OK) return st;
  const Tuple t = to_tuple(*s);
  const Geometry g = geometry(h->info, t, h->grid.nx, h->grid.ny, h->grid.nz);
  info->registers = v->regs;
  info->local_bytes = v->local;
  info->smem_bytes = v->smem;
  info->threads = v->threads;
  info->ctas_per_sm = v->occ;
  info->grid_ctas = (int64_t)g.grid_x * g.grid_y;
  info->compile_s = v->compile_s;
  return CST_OK;
}

// ====================================================================== sweeps
static int64_t numel(const cst_grid& g) {
  return (g.nz + 2 * (int64_t)g.halo) * g.pitch_y * g.pitch_x;
}

static cst_status tmap_for(cst_stencil* h, const double* base, const int box[3],
                           int64_t planes, cst_tmap* out) {
  const std::array<int64_t, 4> key{(int64_t)(uintptr_t)base, box[0], box[1], box[2]};
  auto it = h->tmaps.find(key);
  if (it != h->tmaps.end()) {
    *out = it->second;
    return CST_OK;
  }
  const Driver* d = nullptr;
  cst_status st = driver(&d);
  if (st != CST_OK) return st;
  cst_tmap m;
  const cuuint64_t dims[3] = {(cuuint64_t)h->grid.pitch_x, (cuuint64_t)h->grid.pitch_y,
                              (cuuint64_t)planes};
  const cuuint64_t strides[2] = {(cuuint64_t)h->grid.pitch_x * 8,
                                 (cuuint64_t)h->grid.pitch_x * h->grid.pitch_y * 8};
  const cuuint32_t boxd[3] = {(cuuint32_t)box[0], (cuuint32_t)box[1], (cuuint32_t)box[2]};
  const cuuint32_t estr[3] = {1, 1, 1};
  // L2 promotion of the TMA fetches (experiment hook CST_TMA_PROMO = 0 none, 1 64B,
  // 2 128B, 3 256B; default 256B)
  CUtensorMapL2promotion promo = CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
  if (const char* e = std::getenv("CST_TMA_PROMO")) promo = (CUtensorMapL2promotion)std::atoi(e);
  st = cu_check(d->cuTensorMapEncodeTiled(
                    (CUtensorMap*)&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, (void*)base, dims,
                    strides, boxd, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_NONE, promo,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE),
                "cuTensorMapEncodeTiled");
  if (st != CST_OK) return st;
  h->tmaps[key] = m;
  *out = m;
  return CST_OK;
}

// Launch one sweep of planes [z0, z0 + nz) (local interior z) of the handle's grid.
cst_status cst_launch_range(cst_stencil* h, const cst_setting* s, const double* const* in,
                            double* const* out, int64_t z0, int64_t nzr, cudaStream_t stream,
                            double* const* rout) {
  Variant* v = nullptr;
  cst_status st = get_variant(h, s, &v, rout != nullptr);
  if (st != CST_OK) return st;
  const Driver* d = nullptr;
  st = driver(&d);
  if (st != CST_OK) return st;
  if (nzr <= 0) return CST_OK;
  const Tuple t = to_tuple(*s);
  const cst_grid& G = h->grid;
  const Geometry g = geometry(h->info, t, G.nx, G.ny, nzr);
  if (g.grid_y > 65535) return fail(CST_E_UNSUPPORTED, "grid.y exceeds 65535 (raise SB / TZ)");
  cst_kparams P;
  std::memset(&P, 0, sizeof P);
  const int nin = h->desc.n_inputs, nout = h->desc.n_outputs;
  const int64_t origin = ((int64_t)G.halo * G.pitch_y + G.halo) * G.pitch_x + G.lead_x +
                         z0 * G.pitch_x * G.pitch_y;
  for (int a = 0; a < nin; ++a) {
    P.in[a] = in[a] + origin;
    if (t[F_STAGING] == 3) {
      int box[3] = {g.box[0], g.box[1], g.box[2]};
      if (t[F_STREAM] == 2 && hyp_trimmed(h->info.kind, t)) {  // per-array halos (HTRIM)
        int64_t wa, wb;
        stream_array_box(h->info.kind, h->info.r, t, a, &wa, &wb);
        box[0] = (int)wa;
        box[t[F_SD] == 3 ? 1 : 2] = (int)wb;
      }
      st = tmap_for(h, in[a], box, G.nz + 2 * (int64_t)G.halo, &P.tma[a]);
      if (st != CST_OK) return st;
    }
  }
  for (int o = 0; o < nout; ++o) P.out[o] = out[o] + origin;
  if (rout) {  // the CST_REMOTE twin of the variant reads these
    P.remote = 1;
    for (int o = 0; o < nout; ++o) P.rout[o] = rout[o];
  }
  for (size_t i = 0; i < h->kcoef.size() && i < CST_MAX_COEF; ++i) P.coef[i] = h->kcoef[i];
  P.py = G.pitch_x;
  P.pz = G.pitch_x * G.pitch_y;
  P.nx = (int)G.nx;
  P.ny = (int)G.ny;
  P.nz = (int)nzr;
  P.tox = G.lead_x;
  P.toy = G.halo;
  P.toz = (int)(G.halo + z0);
  P.tiles_a = g.tiles_a;
  P.tiles_b = g.tiles_b;
  P.tiles_c = g.tiles_c;
  P.chunks = g.chunks;
  void* args[] = {&P};
  st = cu_check(d->cuLaunchKernel(v->fn, g.grid_x, g.grid_y, 1, g.threads, 1, 1,
                                  (unsigned)v->smem, (CUstream)stream, args, nullptr),
                "cuLaunchKernel");
  if (st != CST_OK) return st;
  ++h->last_launches;
  return CST_OK;
}

namespace cst {
std::vector<int> pass_schedule(int nsteps, int bt) {
  std::vector<int> v;
  if (bt < 1) bt = 1;
  for (int rem = nsteps; rem > 0;) {
    int b = bt;
    while (b > rem) b /= 2;
    v.push_back(b);
    rem -= b;
  }
  if ((int)(v.size() & 1) != (nsteps & 1)) {
    // one pass more: split the last pass of >= 2 steps in halves (exists: an all-ones
    // schedule has nsteps passes)
    for (int k = (int)v.size() - 1; k >= 0; --k)
      if (v[k] >= 2) {
        v[k] /= 2;
        v.insert(v.begin() + k + 1, v[k]);
        break;
      }
  }
  return v;
}
}  // namespace cst

static bool overlaps(const double* a, const double* b, int64_t n) {
  return a < b + n && b < a + n;
}

extern "C" cst_status cst_sweep(cst_stencil* h, const cst_setting* s, const double* const* in,
                                double* const* out, int32_t nsteps, void* stream) {
  if (!h || !s || !in || !out) return fail(CST_E_INVALID, "null argument");
  if (nsteps < 1) return fail(CST_E_INVALID, "nsteps < 1");
  {
    const Driver* d = nullptr;
    cst_status st = driver(&d);
    if (st != CST_OK) return st;
    CST_CUDA(cudaSetDevice(h->device));
  }
  const int nin = h->desc.n_inputs, nout = h->desc.n_outputs;
  if (nsteps > 1 && nin != nout)
    return fail(CST_E_INVALID, "nsteps > 1 needs n_inputs == n_outputs (ping-pong)");
  const int64_t n = numel(h->grid);
  for (int a = 0; a < nin; ++a) {
    if (!in[a]) return fail(CST_E_INVALID, "null input pointer");
    if ((uintptr_t)in[a] % 256) return fail(CST_E_INVALID, "input pointer not 256-B aligned");
  }
  for (int o = 0; o < nout; ++o) {
    if (!out[o]) return fail(CST_E_INVALID, "null output pointer");
    if ((uintptr_t)out[o] % 256) return fail(CST_E_INVALID, "output pointer not 256-B aligned");
    for (int a = 0; a < nin; ++a)
      if (overlaps(in[a], out[o], n)) return fail(CST_E_INVALID, "input overlaps output");
    for (int q = 0; q < o; ++q)
      if (overlaps(out[q], out[o], n)) return fail(CST_E_INVALID, "outputs overlap");
  }
  {
    const char* rule = check_rules(h->info, to_tuple(*s));
    if (rule) return fail(CST_E_CONSTRAINT, std::string("setting violates ") + rule);
  }
  h->last_launches = 0;
  const double* cur_in[CST_MAX_IN];
  double* cur_out[CST_MAX_OUT];
  for (int a = 0; a < nin; ++a) cur_in[a] = in[a];
  for (int o = 0; o < nout; ++o) cur_out[o] = out[o];
  if (nsteps > 1) {
    // boundary condition of every step = in[]'s halo (reading Q23), every array
    for (int a = 0; a < nin; ++a) {
      cst_status st = copy_halo(h->grid, in[a], out[a], (cudaStream_t)stream);
      if (st != CST_OK) return st;
      ++h->last_launches;
    }
  }
  // temporal blocking: passes of b <= bt fused steps (bt = 1: one launch per step)
  for (int b : pass_schedule(nsteps, s->bt)) {
    cst_setting sp = *s;
    sp.bt = b;
    cst_status st = cst_launch_range(h, &sp, cur_in, cur_out, 0, h->grid.nz, (cudaStream_t)stream);
    if (st != CST_OK) return st;
    if (nsteps > 1)
      for (int a = 0; a < nin; ++a) {  // ping-pong every array (nin == nout here)
        const double* tmp = cur_in[a];
        cur_in[a] = cur_out[a];
        cur_out[a] = const_cast<double*>(tmp);
      }
  }
  return CST_OK;
}

extern "C" int64_t cst_last_launch_count(const cst_stencil* h) { return h ? h->last_launches : 0; }

extern "C" cst_status cst_sync(cst_stencil* h) {
  if (!h) return fail(CST_E_INVALID, "null argument");
  const Driver* d = nullptr;
  cst_status st = driver(&d);
  if (st != CST_OK) return st;
  CST_CUDA(cudaSetDevice(h->device));
  CST_CUDA(cudaDeviceSynchronize());
  CST_CUDA(cudaGetLastError());
  return CST_OK;
}

extern "C" cst_status cst_sweep_host(cst_stencil* h, const cst_setting* s,
                                     const double* const* in, double* const* out,
                                     int32_t nsteps) {
  if (!h || !s || !in || !out) return fail(CST_E_INVALID, "null argument");
  const Driver* d = nullptr;
  cst_status st = driver(&d);
  if (st != CST_OK) return st;
  CST_CUDA(cudaSetDevice(h->device));
  const int nin = h->desc.n_inputs, nout = h->desc.n_outputs;
  const cst_grid& G = h->grid;
  const int64_t n = numel(G);
  if (h->dev_bufs.empty()) {
    for (int i = 0; i < nin + nout; ++i) {
      double* p = nullptr;
      if (cudaMalloc(&p, (size_t)n * sizeof(double)) != cudaSuccess) {
        cudaGetLastError();
        return fail(CST_E_OOM, "cudaMalloc of host-path staging buffers failed");
      }
      h->dev_bufs.push_back(p);
    }
    CST_CUDA(cudaStreamCreateWithFlags(&h->host_stream, cudaStreamNonBlocking));
  }
  cudaStream_t sm = h->host_stream;
  const double* din[CST_MAX_IN];
  double* dout[CST_MAX_OUT];
  for (int a = 0; a < nin; ++a) din[a] = h->dev_bufs[a];
  for (int o = 0; o < nout; ++o) dout[o] = h->dev_bufs[nin + o];
  const int64_t plane = G.pitch_y * G.pitch_x;
  // copy back interior planes [z0, z1) only (halos of host outputs are never written)
  auto copy_back = [&](const double* dsrc, double* hdst, int64_t z0, int64_t z1,
                       cudaStream_t st_) -> cst_status {
    cudaMemcpy3DParms p = {};
    const int64_t first = ((G.halo + z0) * G.pitch_y + G.halo) * G.pitch_x + G.lead_x;
    p.srcPtr = make_cudaPitchedPtr((void*)(dsrc + first), G.pitch_x * 8, G.nx * 8, G.pitch_y);
    p.dstPtr = make_cudaPitchedPtr((void*)(hdst + first), G.pitch_x * 8, G.nx * 8, G.pitch_y);
    p.extent = make_cudaExtent(G.nx * 8, G.ny, z1 - z0);
    p.kind = cudaMemcpyDeviceToHost;
    CST_CUDA(cudaMemcpy3DAsync(&p, st_));
    return CST_OK;
  };
  if (nsteps == 1) {
    cst_setting s1 = *s;  // one step: no temporal blocking
    s1.bt = 1;
    // pipelined along z: H2D of chunk k+1 || sweep of chunk k || D2H of chunk k-1
    if (!h->host_in_stream) {
      CST_CUDA(cudaStreamCreateWithFlags(&h->host_in_stream, cudaStreamNonBlocking));
      CST_CUDA(cudaStreamCreateWithFlags(&h->host_out_stream, cudaStreamNonBlocking));
    }
    // up to 32 chunks of >= max(8, 4r) planes: star25 512^3 25.5 ms vs 26.5 ms with 16 and
    // 30 ms with 8 on B200 (PCIe ~55 GB/s per direction, ~45 GB/s each when both run;
    // tools/e2e_probe.py, profiles/r02/g51_host_chunks.txt)
    const int64_t nc = std::max<int64_t>(
        1, std::min<int64_t>(32, G.nz / std::max<int64_t>(8, 4 * h->info.r)));
    std::vector<cudaEvent_t> evs;
    auto event = [&](cudaStream_t st_) -> cudaEvent_t {
      cudaEvent_t e;
      cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
      cudaEventRecord(e, st_);
      evs.push_back(e);
      return e;
    };
    int64_t copied = 0;  // padded planes already on the device
    const int64_t planes = G.nz + 2 * (int64_t)G.halo;
    // per row only the columns a kernel can read: the interior and an x-halo of halo rounded
    // up to even (the kernels' 16-B aligned TMA boxes), not the row padding (4.4 % of a
    // star25 512^3 row: 520 of 544 doubles)
    const int64_t xh = std::min<int64_t>(G.lead_x, G.halo + (G.halo & 1));
    const int64_t xw = std::min<int64_t>(G.pitch_x - (G.lead_x - xh), G.nx + 2 * xh);
    auto copy_in = [&](const double* hsrc, double* ddst, int64_t p0, int64_t p1) -> cst_status {
      cudaMemcpy3DParms q = {};
      const int64_t first = p0 * plane + (G.lead_x - xh);
      q.srcPtr = make_cudaPitchedPtr((void*)(hsrc + first), G.pitch_x * 8, xw * 8, G.pitch_y);
      q.dstPtr = make_cudaPitchedPtr((void*)(ddst + first), G.pitch_x * 8, xw * 8, G.pitch_y);
      q.extent = make_cudaExtent(xw * 8, G.pitch_y, p1 - p0);
      q.kind = cudaMemcpyHostToDevice;
      CST_CUDA(cudaMemcpy3DAsync(&q, h->host_in_stream));
      return CST_OK;
    };
    h->last_launches = 0;
    st = CST_OK;
    for (int64_t k = 0; k < nc && st == CST_OK; ++k) {
      const int64_t z0 = k * G.nz / nc, z1 = (k + 1) * G.nz / nc;
      const int64_t need = k == nc - 1 ? planes : std::min(planes, z1 + G.halo + h->info.r);
      for (int a = 0; a < nin && need > copied && st == CST_OK; ++a)
        st = copy_in(in[a], h->dev_bufs[a], copied, need);
      if (st != CST_OK) break;
      copied = std::max(copied, need);
      CST_CUDA(cudaStreamWaitEvent(sm, event(h->host_in_stream), 0));
      st = cst_launch_range(h, &s1, din, dout, z0, z1 - z0, sm);
      if (st != CST_OK) break;
      CST_CUDA(cudaStreamWaitEvent(h->host_out_stream, event(sm), 0));
      for (int o = 0; o < nout && st == CST_OK; ++o)
        st = copy_back(dout[o], out[o], z0, z1, h->host_out_stream);
    }
    cudaStreamSynchronize(h->host_in_stream);
    cudaStreamSynchronize(sm);
    cudaStreamSynchronize(h->host_out_stream);
    for (cudaEvent_t e : evs) cudaEventDestroy(e);
    if (st != CST_OK) return st;
    CST_CUDA(cudaGetLastError());
    return CST_OK;
  }
  for (int a = 0; a < nin; ++a)
    CST_CUDA(cudaMemcpyAsync(h->dev_bufs[a], in[a], (size_t)n * 8, cudaMemcpyHostToDevice, sm));
  // (no copy of out[]: cst_sweep gives the output buffer in[]'s halo, the boundary condition)
  st = cst_sweep(h, s, din, dout, nsteps, sm);
  if (st != CST_OK) return st;
  for (int o = 0; o < nout; ++o) {
    st = copy_back(dout[o], out[o], 0, G.nz, sm);
    if (st != CST_OK) return st;
  }
  for (int a = 0; a < nin; ++a) {
    st = copy_back(din[a], const_cast<double*>(in[a]), 0, G.nz, sm);
    if (st != CST_OK) return st;
  }
  CST_CUDA(cudaStreamSynchronize(sm));
  CST_CUDA(cudaGetLastError());
  return CST_OK;
}

extern "C" cst_status cst_time_setting(cst_stencil* h, const cst_setting* s,
                                       const double* const* in, double* const* out,
                                       int32_t nsteps, int32_t warmup, int32_t reps,
                                       void* stream, double* ms) {
  if (!h || !s || !ms || reps < 1 || nsteps < 1) return fail(CST_E_INVALID, "bad argument");
  const Driver* d = nullptr;
  cst_status st = driver(&d);
  if (st != CST_OK) return st;
  CST_CUDA(cudaSetDevice(h->device));
  cudaStream_t sm = (cudaStream_t)stream;
  for (int i = 0; i < warmup; ++i) {
    st = cst_sweep(h, s, in, out, nsteps, sm);
    if (st != CST_OK) return st;
  }
  std::vector<cudaEvent_t> ev(reps + 1);
  for (auto& e : ev) CST_CUDA(cudaEventCreate(&e));
  CST_CUDA(cudaEventRecord(ev[0], sm));
  for (int i = 0; i < reps; ++i) {
    st = cst_sweep(h, s, in, out, nsteps, sm);
    if (st != CST_OK) break;
    CST_CUDA(cudaEventRecord(ev[i + 1], sm));
  }
  if (st != CST_OK) {
    for (auto& e : ev) cudaEventDestroy(e);
    return st;
  }
  CST_CUDA(cudaEventSynchronize(ev[reps]));
  cudaError_t ke = cudaGetLastError();
  std::vector<double> t(reps);
  for (int i = 0; i < reps; ++i) {
    float f = 0;
    cudaEventElapsedTime(&f, ev[i], ev[i + 1]);
    t[i] = f;
  }
  for (auto& e : ev) cudaEventDestroy(e);
  if (ke != cudaSuccess) return fail(CST_E_CUDA, std::string("kernel: ") + cudaGetErrorString(ke));
  std::sort(t.begin(), t.end());
  *ms = (reps % 2 ? t[reps / 2] : 0.5 * (t[reps / 2 - 1] + t[reps / 2])) / nsteps;
  return CST_OK;
}
