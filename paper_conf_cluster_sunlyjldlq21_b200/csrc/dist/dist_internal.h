// dist_internal.h — the cst_dist handle, shared by dist.cpp (z-slab sweeps, halo
// transports) and dist_tune.cpp (population-parallel tuning).
#ifndef CST_DIST_INTERNAL_H
#define CST_DIST_INTERNAL_H
#include "../runtime/internal.h"

#ifdef CST_HAVE_NCCL
#include <nccl.h>
#endif

enum { F_BND_LO = 0, F_BND_HI = 1, F_DONE_LO = 2, F_DONE_HI = 3, F_WORDS = 16 };

struct P2PPeer {
  bool open = false;
  double* buf[2][CST_MAX_IN] = {};  // the peer's ping-pong buffers (a, b), mapped here
  unsigned long long* flags = nullptr;  // the peer's flag words, mapped here
  std::vector<void*> bases;             // IPC mappings to close
};

struct cst_dist {
  cst_stencil* h = nullptr;
  int32_t nranks = 1, rank = 0;
  cudaStream_t s_comm = nullptr;
  cudaEvent_t ev_bnd = nullptr, ev_comm = nullptr;
#ifdef CST_HAVE_NCCL
  ncclComm_t comm = nullptr;
#endif
  // peer-memory transport
  bool p2p = false;
  unsigned long long* flags = nullptr;  // my flag words (F_WORDS x u64)
  const double* mine[2][CST_MAX_IN] = {};  // my registered ping-pong buffers (a, b)
  bool exported = false;
  P2PPeer lo, hi;                        // rank - 1, rank + 1
  unsigned long long epoch = 0;
  bool broken = false;  // a step failed after its epoch was published: peers cannot resync
  // population-parallel tuning (dist_tune.cpp): caller-supplied host collectives, or NCCL
  bool host_only = false;  // cst_dist_create_host: no device resources, tuning only
  cst_collectives coll{};
  bool has_coll = false;
};


#endif
