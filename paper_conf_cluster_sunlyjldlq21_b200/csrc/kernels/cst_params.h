// cst_params.h — kernel parameter block shared by the host runtime (g++/nvcc) and the
// run-time compiled kernels (NVRTC).  Plain C layout; no library headers.
#ifndef CST_PARAMS_H
#define CST_PARAMS_H

#define CST_MAX_IN 8
#define CST_MAX_OUT 5
#define CST_MAX_COEF 27

// Opaque CUtensorMap (128 bytes, 64-byte aligned), filled by cuTensorMapEncodeTiled.
struct __attribute__((aligned(64))) cst_tmap {
  unsigned long long opaque[16];
};

// Passed by value as `const __grid_constant__ cst_kparams` (TMA descriptors must live in
// parameter / constant / global memory).
struct __attribute__((aligned(64))) cst_kparams {
  cst_tmap tma[CST_MAX_IN];          // one 3-D map per input over the whole allocation
  const double* in[CST_MAX_IN];      // &element(0,0,0) of the (sub)domain, per input
  double* out[CST_MAX_OUT];          // &element(0,0,0) of the (sub)domain, per output
  double coef[CST_MAX_COEF];         // used when use_constant == 1 (param constant bank)
  long long py;                      // element stride of y  (= pitch_x)
  long long pz;                      // element stride of z  (= pitch_x * pitch_y)
  int nx, ny, nz;                    // interior extents of the (sub)domain
  int tox, toy, toz;                 // TMA coordinates of element (0,0,0)
  int tiles_a, tiles_b;              // CTA tiles over the two non-streamed dims (or x,y)
  int tiles_c;                       // third tile dim (non-streaming z tiles)
  int chunks;                        // streaming chunks (SB)
  int remote;                        // 1: every store also goes to rout[q] + same offset
  double* rout[CST_MAX_OUT];         // peer-mapped neighbour halo (fused z-slab exchange)
};

#endif
