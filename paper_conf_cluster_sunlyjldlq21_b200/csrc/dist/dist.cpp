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

#include "../runtime/internal.h"

#ifdef CST_HAVE_NCCL
#include <nccl.h>
#endif

struct cst_dist {
  cst_stencil* h = nullptr;
  int32_t nranks = 1, rank = 0;
  cudaStream_t s_comm = nullptr;
  cudaEvent_t ev_bnd = nullptr, ev_comm = nullptr;
#ifdef CST_HAVE_NCCL
  ncclComm_t comm = nullptr;
#endif
};

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
  if (nranks > 1) {
#ifdef CST_HAVE_NCCL
    if (!uid) {
      delete D;
      return fail(CST_E_INVALID, "nccl_unique_id required for nranks > 1");
    }
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
#ifdef CST_HAVE_NCCL
  if (D->comm) ncclCommDestroy(D->comm);
#endif
  if (D->s_comm) cudaStreamDestroy(D->s_comm);
  if (D->ev_bnd) cudaEventDestroy(D->ev_bnd);
  if (D->ev_comm) cudaEventDestroy(D->ev_comm);
  delete D;
}

extern "C" cst_status cst_dist_sweep(cst_dist* D, const cst_setting* s, const double* const* in,
                                     double* const* out, int32_t nsteps, void* stream) {
  if (!D || !s || !in || !out) return fail(CST_E_INVALID, "null argument");
  if (nsteps < 1) return fail(CST_E_INVALID, "nsteps < 1");
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
  if (nsteps > 1)  // boundary condition of every step = in[]'s halo (as cst_sweep)
    for (int a = 0; a < nio; ++a) {
      st = copy_halo(G, in[a], out[a], sc);
      if (st != CST_OK) return st;
    }
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
    for (int i = 0; i < nslabs * nio && st == CST_OK; ++i) st = copy_halo(G, in_slabs[i], out_slabs[i], sc);
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
