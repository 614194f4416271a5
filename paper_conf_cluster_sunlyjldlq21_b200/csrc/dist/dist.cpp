// dist.cpp — z-slab domain decomposition of the sweep (north_star: "a z-slab
// domain decomposition with NCCL halo exchange over NVLink, overlapped with the interior
// sweep").  Per step, on the caller's compute stream:
//   1. boundary planes [0, r) and [nz-r, nz) of this rank's output          (kernel)
//   2. event -> communication stream: grouped ncclSend/ncclRecv of r contiguous planes
//      to/from rank-1 and rank+1 into the output's halo planes               (NCCL, NVLink)
//   3. concurrently, the interior planes [r, nz-r)                            (kernel)
//   4. compute stream waits for the exchange; in/out ping-pong for nsteps > 1
// z is the slowest dimension, so every transfer is one contiguous block (zero-copy).
// Every point's summation order is independent of the launch's z-range, so the slab
// result is bit-identical to the single-GPU sweep with the same setting.
#include <cstring>

#include "dist_internal.h"

// Fused halo exchange over peer memory: no NCCL.  The boundary
// launches store every edge-plane value both locally and, through a CUDA IPC mapping of
// the neighbour's matching buffer, straight into the neighbour's halo (NVLink / NVSwitch
// stores on a multi-GPU node).  Steps are ordered by 64-bit flag words each rank keeps in
// its own device memory and its neighbours write over the same mappings:
//   BND_LO / BND_HI   epoch of the last step whose boundary stores the lower / upper
//                     neighbour has completed into my halo                       (RAW)
//   DONE_LO / DONE_HI epoch of the last step the lower / upper neighbour has finished
//                     (it no longer reads the buffer my next boundary launch writes) (WAR)
// Per step (epoch e, one stream):  wait DONE >= e-1 | boundary launches with remote stores
// | signal BND = e | interior | signal DONE = e | wait BND >= e.  Waits spin on an acquire
// load with a 30 s bound (then trap: a dead peer is an error, not a hang).
using namespace cst;

extern "C" cst_status cst_dist_halo_plan(int32_t nranks, int32_t rank, int64_t nz, int32_t r,
                                         cst_halo_xfer* x, int32_t* n) {
  if (!x || !n) return fail(CST_E_INVALID, "null argument");
  if (nranks < 1 || rank < 0 || rank >= nranks || r < 1)
    return fail(CST_E_INVALID, "bad nranks / rank / r");
  if (nz < 2 * (int64_t)r)
    return fail(CST_E_INVALID, "z-slab needs nz >= 2r local planes (boundary/interior split)");
  int k = 0;
  // order: the lower neighbour first, sends before receives (grouped anyway)
  if (rank > 0) {
    x[k++] = cst_halo_xfer{rank - 1, 1, 0, r};
    x[k++] = cst_halo_xfer{rank - 1, 0, -(int64_t)r, r};
  }
  if (rank < nranks - 1) {
    x[k++] = cst_halo_xfer{rank + 1, 1, nz - r, r};
    x[k++] = cst_halo_xfer{rank + 1, 0, nz, r};
  }
  *n = k;
  return CST_OK;
}

static int64_t plane_offset(const cst_grid& g, int64_t z) {
  return (z + g.halo) * g.pitch_y * g.pitch_x;
}

#ifdef CST_HAVE_NCCL
static cst_status nccl_check(ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return CST_OK;
  return fail(CST_E_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}
#endif

extern "C" cst_status cst_dist_nccl_unique_id(void* id128) {
  if (!id128) return fail(CST_E_INVALID, "null argument");
#ifdef CST_HAVE_NCCL
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  ncclUniqueId id;
  cst_status st = nccl_check(ncclGetUniqueId(&id), "ncclGetUniqueId");
  if (st != CST_OK) return st;
  std::memcpy(id128, &id, 128);
  return CST_OK;
#else
  return fail(CST_E_UNSUPPORTED, "libcst built without NCCL");
#endif
}

extern "C" cst_status cst_dist_create(cst_stencil* h, int32_t nranks, int32_t rank,
                                      const void* uid, cst_dist** out) {
  if (!h || !out) return fail(CST_E_INVALID, "null argument");
  cst_halo_xfer x[4];
  int32_t n = 0;
  cst_status st = cst_dist_halo_plan(nranks, rank, h->grid.nz, h->desc.order, x, &n);
  if (st != CST_OK) return st;
  if (h->desc.n_inputs != h->desc.n_outputs)
    return fail(CST_E_UNSUPPORTED, "z-slab sweeps need n_inputs == n_outputs (ping-pong)");
  if (h->grid.halo != h->desc.order)
    return fail(CST_E_INVALID, "z-slab exchange needs grid.halo == order");
  const Driver* d = nullptr;
  st = driver(&d);
  if (st != CST_OK) return st;
  CST_CUDA(cudaSetDevice(h->device));
  auto* D = new cst_dist();
  D->h = h;
  D->nranks = nranks;
  D->rank = rank;
  cudaStreamCreateWithPriority(&D->s_comm, cudaStreamNonBlocking, -1);
  cudaEventCreateWithFlags(&D->ev_bnd, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&D->ev_comm, cudaEventDisableTiming);
  if (nranks > 1 && !uid) {  // fused peer-memory transport
    D->p2p = true;
    if (cudaMalloc(&D->flags, F_WORDS * sizeof(unsigned long long)) != cudaSuccess ||
        cudaMemset(D->flags, 0, F_WORDS * sizeof(unsigned long long)) != cudaSuccess) {
      cudaGetLastError();
      delete D;
      return fail(CST_E_OOM, "p2p flag words");
    }
  } else if (nranks > 1) {
#ifdef CST_HAVE_NCCL
    ncclUniqueId id;
    std::memcpy(&id, uid, 128);
    st = nccl_check(ncclCommInitRank(&D->comm, nranks, id, rank), "ncclCommInitRank");
    if (st != CST_OK) {
      delete D;
      return st;
    }
#else
    delete D;
    return fail(CST_E_UNSUPPORTED, "libcst built without NCCL");
#endif
  }
  *out = D;
  return CST_OK;
}

extern "C" void cst_dist_destroy(cst_dist* D) {
  if (!D) return;
  if (D->p2p) {
    cudaSetDevice(D->h->device);
    cudaDeviceSynchronize();
    for (P2PPeer* p : {&D->lo, &D->hi})
      for (void* b : p->bases) cudaIpcCloseMemHandle(b);
    if (D->flags) cudaFree(D->flags);
  }
#ifdef CST_HAVE_NCCL
  if (D->comm) ncclCommDestroy(D->comm);
#endif
  if (D->s_comm) cudaStreamDestroy(D->s_comm);
  if (D->ev_bnd) cudaEventDestroy(D->ev_bnd);
  if (D->ev_comm) cudaEventDestroy(D->ev_comm);
  delete D;
}

// ---------------------------------------------------------------- peer-memory transport
namespace {
struct P2PBlob {
  uint64_t magic;
  int32_t nio, rank, nranks, device;
  // geometry: the remote store offsets are computed from the LOCAL grid, so the peer's
  // must be identical (a mismatch would put peer stores at wrong offsets)
  int64_t nx, ny, nz, pitch_x, pitch_y;
  int32_t halo, lead_x, order, kind;
  cudaIpcMemHandle_t buf[2][CST_MAX_IN];
  int64_t off[2][CST_MAX_IN];
  cudaIpcMemHandle_t flags;
  int64_t flags_off;
};
static_assert(sizeof(P2PBlob) <= CST_P2P_BLOB_BYTES, "blob size");
const uint64_t kBlobMagic = 0x43535450325032ULL;  // "CSTP2P2"

cst_status ipc_handle(const void* p, cudaIpcMemHandle_t* hd, int64_t* off) {
  const Driver* d = nullptr;
  cst_status st = driver(&d);
  if (st != CST_OK) return st;
  CUdeviceptr base = 0;
  size_t size = 0;
  st = cu_check(d->cuMemGetAddressRange(&base, &size, (CUdeviceptr)p), "cuMemGetAddressRange");
  if (st != CST_OK) return st;
  CST_CUDA(cudaIpcGetMemHandle(hd, (void*)base));
  *off = (int64_t)((CUdeviceptr)p - base);
  return CST_OK;
}
}  // namespace

extern "C" cst_status cst_dist_p2p_export(cst_dist* D, double* const* buf_a,
                                          double* const* buf_b, void* blob) {
  if (!D || !buf_a || !buf_b || !blob) return fail(CST_E_INVALID, "null argument");
  if (!D->p2p) return fail(CST_E_INVALID, "handle was created for NCCL (nccl_unique_id given)");
  CST_CUDA(cudaSetDevice(D->h->device));
  const int nio = D->h->desc.n_inputs;
  P2PBlob b;
  std::memset(&b, 0, sizeof b);
  b.magic = kBlobMagic;
  b.nio = nio;
  b.rank = D->rank;
  b.nranks = D->nranks;
  b.device = D->h->device;
  const cst_grid& G = D->h->grid;
  b.nx = G.nx;
  b.ny = G.ny;
  b.nz = G.nz;
  b.pitch_x = G.pitch_x;
  b.pitch_y = G.pitch_y;
  b.halo = G.halo;
  b.lead_x = G.lead_x;
  b.order = D->h->desc.order;
  b.kind = D->h->desc.kind;
  for (int a = 0; a < nio; ++a) {
    if (!buf_a[a] || !buf_b[a]) return fail(CST_E_INVALID, "null buffer");
    cst_status st = ipc_handle(buf_a[a], &b.buf[0][a], &b.off[0][a]);
    if (st == CST_OK) st = ipc_handle(buf_b[a], &b.buf[1][a], &b.off[1][a]);
    if (st != CST_OK) return st;
    D->mine[0][a] = buf_a[a];
    D->mine[1][a] = buf_b[a];
  }
  cst_status st = ipc_handle(D->flags, &b.flags, &b.flags_off);
  if (st != CST_OK) return st;
  std::memset(blob, 0, CST_P2P_BLOB_BYTES);
  std::memcpy(blob, &b, sizeof b);
  D->exported = true;
  return CST_OK;
}

extern "C" cst_status cst_dist_p2p_import(cst_dist* D, int32_t peer, const void* blob) {
  if (!D || !blob) return fail(CST_E_INVALID, "null argument");
  if (!D->p2p) return fail(CST_E_INVALID, "handle was created for NCCL (nccl_unique_id given)");
  if (peer != D->rank - 1 && peer != D->rank + 1)
    return fail(CST_E_INVALID, "p2p peers are rank - 1 and rank + 1");
  if (peer < 0 || peer >= D->nranks) return fail(CST_E_INVALID, "peer out of range");
  P2PBlob b;
  std::memcpy(&b, blob, sizeof b);
  if (b.magic != kBlobMagic || b.nio != D->h->desc.n_inputs || b.rank != peer ||
      b.nranks != D->nranks)
    return fail(CST_E_INVALID, "p2p blob does not belong to this decomposition / peer");
  {
    const cst_grid& G = D->h->grid;
    if (b.nx != G.nx || b.ny != G.ny || b.nz != G.nz || b.pitch_x != G.pitch_x ||
        b.pitch_y != G.pitch_y || b.halo != G.halo || b.lead_x != G.lead_x ||
        b.order != D->h->desc.order || b.kind != D->h->desc.kind)
      return fail(CST_E_INVALID, "p2p blob: the peer's grid geometry / stencil differs from "
                                 "mine (nx, ny, nz, pitches, halo, lead_x, order, kind must match)");
  }
  CST_CUDA(cudaSetDevice(D->h->device));
  P2PPeer& P = peer < D->rank ? D->lo : D->hi;
  for (void* base : P.bases) cudaIpcCloseMemHandle(base);
  P = P2PPeer();
  auto open = [&](const cudaIpcMemHandle_t& hd, int64_t off, void** out) -> cst_status {
    void* base = nullptr;
    // one mapping per allocation: buffers that share one (e.g. a caching allocator's
    // block) come back as the same base pointer
    CST_CUDA(cudaIpcOpenMemHandle(&base, hd, cudaIpcMemLazyEnablePeerAccess));
    P.bases.push_back(base);
    *out = (char*)base + off;
    return CST_OK;
  };
  for (int a = 0; a < b.nio; ++a)
    for (int r = 0; r < 2; ++r) {
      void* p = nullptr;
      cst_status st = open(b.buf[r][a], b.off[r][a], &p);
      if (st != CST_OK) return st;
      P.buf[r][a] = (double*)p;
    }
  void* f = nullptr;
  cst_status st = open(b.flags, b.flags_off, &f);
  if (st != CST_OK) return st;
  P.flags = (unsigned long long*)f;
  P.open = true;
  return CST_OK;
}

static cst_status dist_sweep_p2p(cst_dist* D, const cst_setting* s, const double* const* in,
                                 double* const* out, int32_t nsteps, cudaStream_t sc) {
  cst_stencil* h = D->h;
  const cst_grid& G = h->grid;
  const int r = h->desc.order;
  const int nio = h->desc.n_inputs;
  const bool has_lo = D->rank > 0, has_hi = D->rank < D->nranks - 1;
  if (!D->exported || (has_lo && !D->lo.open) || (has_hi && !D->hi.open))
    return fail(CST_E_INVALID, "p2p transport: export my buffers and import both neighbours first");
  // which registered buffer set is in[]: role 0 = a, 1 = b
  int role = -1;
  for (int c = 0; c < 2 && role < 0; ++c) {
    bool ok = true;
    for (int a = 0; a < nio; ++a)
      ok = ok && in[a] == D->mine[c][a] && out[a] == D->mine[1 - c][a];
    if (ok) role = c;
  }
  if (role < 0)
    return fail(CST_E_INVALID, "p2p transport: in/out must be the exported buffer sets (a, b)");
  if (D->broken)
    return fail(CST_E_INTERNAL, "p2p transport: an earlier step failed mid-protocol; the "
                                "ranks cannot resynchronise (destroy and recreate the handle)");
  // every variant this protocol launches is resolved before any epoch is published: a
  // compile / R13 / load failure must not leave the neighbours waiting for this rank
  {
    cst_status st = cst_resolve_variant(h, s, has_lo || has_hi);
    if (st != CST_OK) return st;
  }
  const int64_t pz = G.pitch_x * G.pitch_y;
  const int64_t origin0 = ((int64_t)G.halo * G.pitch_y + G.halo) * G.pitch_x + G.lead_x;
  const double* cin[CST_MAX_IN];
  double* cout[CST_MAX_OUT];
  for (int a = 0; a < nio; ++a) {
    cin[a] = in[a];
    cout[a] = out[a];
  }
  h->last_launches = 0;
  int64_t extra = 0;  // signal / wait kernels
  for (int step = 0; step < nsteps; ++step) {
    const int orole = 1 - role;  // role of this step's output buffers
    const unsigned long long e = ++D->epoch;
    // WAR: both neighbours finished step e-1 (they read the buffers my stores target)
    cst_status st = p2p_wait(sc, has_lo ? D->flags + F_DONE_LO : nullptr, e - 1,
                             has_hi ? D->flags + F_DONE_HI : nullptr, e - 1);
    if (st != CST_OK) return D->broken = true, st;
    ++extra;
    // boundary planes: local stores + the same values into the neighbours' halos
    double* rlo[CST_MAX_OUT];
    double* rhi[CST_MAX_OUT];
    for (int a = 0; a < nio; ++a) {
      rlo[a] = has_lo ? D->lo.buf[orole][a] + origin0 + G.nz * pz : nullptr;
      rhi[a] = has_hi ? D->hi.buf[orole][a] + origin0 - (int64_t)r * pz : nullptr;
    }
    st = cst_launch_range(h, s, cin, cout, 0, r, sc, has_lo ? rlo : nullptr);
    if (st != CST_OK) return D->broken = true, st;
    if (G.nz > r) {
      st = cst_launch_range(h, s, cin, cout, G.nz - r, r, sc, has_hi ? rhi : nullptr);
      if (st != CST_OK) return D->broken = true, st;
    }
    // my boundary stores are in the neighbours' halos: lower neighbour's BND_HI, upper's BND_LO
    st = p2p_signal(sc, has_lo ? D->lo.flags + F_BND_HI : nullptr,
                    has_hi ? D->hi.flags + F_BND_LO : nullptr, e);
    if (st != CST_OK) return D->broken = true, st;
    ++extra;
    if (G.nz > 2 * r) {
      st = cst_launch_range(h, s, cin, cout, r, G.nz - 2 * r, sc);
      if (st != CST_OK) return D->broken = true, st;
    }
    st = p2p_signal(sc, has_lo ? D->lo.flags + F_DONE_HI : nullptr,
                    has_hi ? D->hi.flags + F_DONE_LO : nullptr, e);
    if (st != CST_OK) return D->broken = true, st;
    // RAW: the neighbours' boundary stores of this step are in my output halo
    st = p2p_wait(sc, has_lo ? D->flags + F_BND_LO : nullptr, e,
                  has_hi ? D->flags + F_BND_HI : nullptr, e);
    if (st != CST_OK) return D->broken = true, st;
    extra += 2;
    if (nsteps > 1) {
      for (int a = 0; a < nio; ++a) {
        const double* t = cin[a];
        cin[a] = cout[a];
        cout[a] = const_cast<double*>(t);
      }
      role = 1 - role;
    }
  }
  h->last_launches += extra;
  return CST_OK;
}

extern "C" cst_status cst_dist_sweep(cst_dist* D, const cst_setting* s, const double* const* in,
                                     double* const* out, int32_t nsteps, void* stream) {
  if (!D || !s || !in || !out) return fail(CST_E_INVALID, "null argument");
  if (nsteps < 1) return fail(CST_E_INVALID, "nsteps < 1");
  if (D->host_only) return fail(CST_E_INVALID, "a cst_dist_create_host handle only tunes");
  cst_stencil* h = D->h;
  const cst_grid& G = h->grid;
  const int r = h->desc.order;
  const int nio = h->desc.n_inputs;
  cudaStream_t sc = (cudaStream_t)stream;
  CST_CUDA(cudaSetDevice(h->device));
  cst_halo_xfer x[4];
  int32_t nx = 0;
  cst_status st = cst_dist_halo_plan(D->nranks, D->rank, G.nz, r, x, &nx);
  if (st != CST_OK) return st;
  const size_t count = (size_t)r * G.pitch_y * G.pitch_x;
  const double* cin[CST_MAX_IN];
  double* cout[CST_MAX_OUT];
  for (int a = 0; a < nio; ++a) {
    cin[a] = in[a];
    cout[a] = out[a];
  }
  if (s->bt > 1)
    return fail(CST_E_UNSUPPORTED, "temporal blocking (bt > 1) needs bt*order halo planes; "
                                   "cst_dist_sweep exchanges order planes per step");
  if (nsteps > 1)  // boundary condition of every step = in[]'s halo (as cst_sweep); of
                   // the z-halo planes facing a neighbour only the x/y ring is copied — their
                   // interior x/y is the exchange's (the peer may already be storing into it)
    for (int a = 0; a < nio; ++a) {
      st = copy_halo(G, in[a], out[a], sc, D->rank == 0, D->rank == D->nranks - 1);
      if (st != CST_OK) return st;
    }
  if (D->p2p) return dist_sweep_p2p(D, s, in, out, nsteps, sc);
  h->last_launches = 0;  // cst_launch_range counts every launch
  for (int step = 0; step < nsteps; ++step) {
    // 1. boundary planes first
    st = cst_launch_range(h, s, cin, cout, 0, r, sc);
    if (st != CST_OK) return st;
    if (G.nz > r) {
      st = cst_launch_range(h, s, cin, cout, G.nz - r, r, sc);
      if (st != CST_OK) return st;
    }
    // 2. exchange on the communication stream
    if (D->nranks > 1) {
      CST_CUDA(cudaEventRecord(D->ev_bnd, sc));
      CST_CUDA(cudaStreamWaitEvent(D->s_comm, D->ev_bnd, 0));
#ifdef CST_HAVE_NCCL
      st = nccl_check(ncclGroupStart(), "ncclGroupStart");
      if (st != CST_OK) return st;
      for (int a = 0; a < nio; ++a)
        for (int i = 0; i < nx; ++i) {
          double* p = cout[a] + plane_offset(G, x[i].plane_begin);
          const ncclResult_t rr =
              x[i].is_send ? ncclSend(p, count, ncclDouble, x[i].peer, D->comm, D->s_comm)
                           : ncclRecv(p, count, ncclDouble, x[i].peer, D->comm, D->s_comm);
          if (rr != ncclSuccess) {
            ncclGroupEnd();
            return nccl_check(rr, x[i].is_send ? "ncclSend" : "ncclRecv");
          }
        }
      st = nccl_check(ncclGroupEnd(), "ncclGroupEnd");
      if (st != CST_OK) return st;
#endif
      CST_CUDA(cudaEventRecord(D->ev_comm, D->s_comm));
    }
    // 3. interior concurrently
    if (G.nz > 2 * r) {
      st = cst_launch_range(h, s, cin, cout, r, G.nz - 2 * r, sc);
      if (st != CST_OK) return st;
    }
    // 4. next step (or the caller) sees the exchanged halos
    if (D->nranks > 1) CST_CUDA(cudaStreamWaitEvent(sc, D->ev_comm, 0));
    if (nsteps > 1)
      for (int a = 0; a < nio; ++a) {
        const double* t = cin[a];
        cin[a] = cout[a];
        cout[a] = const_cast<double*>(t);
      }
  }
  return CST_OK;
}

// One process drives all slabs of a z-decomposition on the handle's device; halos move
// with cudaMemcpyAsync on a second stream, mirroring cst_dist_sweep step for step.  Tests
// the decomposition on one GPU (NCCL forbids two ranks on one device).
extern "C" cst_status cst_dist_sweep_loopback(cst_stencil* h, int32_t nslabs, const cst_setting* s,
                                              double* const* in_slabs, double* const* out_slabs,
                                              int32_t nsteps, void* stream) {
  if (!h || !s || !in_slabs || !out_slabs) return fail(CST_E_INVALID, "null argument");
  if (nslabs < 1 || nsteps < 1) return fail(CST_E_INVALID, "nslabs / nsteps < 1");
  if (h->desc.n_inputs != h->desc.n_outputs)
    return fail(CST_E_UNSUPPORTED, "z-slab sweeps need n_inputs == n_outputs");
  if (h->grid.halo != h->desc.order)
    return fail(CST_E_INVALID, "z-slab exchange needs grid.halo == order");
  const cst_grid& G = h->grid;
  const int r = h->desc.order;
  const int nio = h->desc.n_inputs;
  const Driver* d = nullptr;
  cst_status st = driver(&d);
  if (st != CST_OK) return st;
  CST_CUDA(cudaSetDevice(h->device));
  cudaStream_t sc = (cudaStream_t)stream, sx = nullptr;
  cudaEvent_t e1 = nullptr, e2 = nullptr;
  CST_CUDA(cudaStreamCreateWithFlags(&sx, cudaStreamNonBlocking));
  CST_CUDA(cudaEventCreateWithFlags(&e1, cudaEventDisableTiming));
  CST_CUDA(cudaEventCreateWithFlags(&e2, cudaEventDisableTiming));
  const size_t bytes = (size_t)r * G.pitch_y * G.pitch_x * sizeof(double);
  std::vector<const double*> cin(nslabs * nio);
  std::vector<double*> cout(nslabs * nio);
  for (int i = 0; i < nslabs * nio; ++i) {
    cin[i] = in_slabs[i];
    cout[i] = out_slabs[i];
  }
  if (s->bt > 1) st = fail(CST_E_UNSUPPORTED, "temporal blocking (bt > 1) is not supported by z-slab sweeps");
  if (nsteps > 1)  // boundary condition of every step = in[]'s halo (as cst_sweep)
    for (int i = 0; i < nslabs * nio && st == CST_OK; ++i)
      st = copy_halo(G, in_slabs[i], out_slabs[i], sc, i / nio == 0, i / nio == nslabs - 1);
  h->last_launches = 0;  // cst_launch_range counts every launch
  for (int step = 0; step < nsteps && st == CST_OK; ++step) {
    for (int k = 0; k < nslabs && st == CST_OK; ++k) {
      st = cst_launch_range(h, s, &cin[k * nio], &cout[k * nio], 0, r, sc);
      if (st == CST_OK && G.nz > r)
        st = cst_launch_range(h, s, &cin[k * nio], &cout[k * nio], G.nz - r, r, sc);
    }
    if (st != CST_OK) break;
    cudaEventRecord(e1, sc);
    cudaStreamWaitEvent(sx, e1, 0);
    for (int k = 0; k < nslabs; ++k) {
      cst_halo_xfer x[4];
      int32_t nx = 0;
      st = cst_dist_halo_plan(nslabs, k, G.nz, r, x, &nx);
      if (st != CST_OK) break;
      for (int i = 0; i < nx; ++i) {
        if (!x[i].is_send) continue;
        // the receiver's matching halo: lower neighbour receives into [nz, nz+r), upper into [-r, 0)
        const int64_t dst_plane = x[i].peer < k ? G.nz : -(int64_t)r;
        for (int a = 0; a < nio; ++a)
          cudaMemcpyAsync(cout[x[i].peer * nio + a] + plane_offset(G, dst_plane),
                          cout[k * nio + a] + plane_offset(G, x[i].plane_begin), bytes,
                          cudaMemcpyDeviceToDevice, sx);
      }
    }
    cudaEventRecord(e2, sx);
    for (int k = 0; k < nslabs && st == CST_OK && G.nz > 2 * r; ++k)
      st = cst_launch_range(h, s, &cin[k * nio], &cout[k * nio], r, G.nz - 2 * r, sc);
    cudaStreamWaitEvent(sc, e2, 0);
    if (nsteps > 1)
      for (int i = 0; i < nslabs * nio; ++i) {
        const double* t = cin[i];
        cin[i] = cout[i];
        cout[i] = const_cast<double*>(t);
      }
  }
  cudaStreamSynchronize(sx);
  cudaStreamDestroy(sx);
  cudaEventDestroy(e1);
  cudaEventDestroy(e2);
  if (st != CST_OK) return st;
  CST_CUDA(cudaGetLastError());
  return CST_OK;
}
