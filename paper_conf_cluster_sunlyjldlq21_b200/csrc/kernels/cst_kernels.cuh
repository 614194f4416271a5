// cst_kernels.cuh — the sm_100a complex-stencil sweep kernel family.
//
// Compiled at run time by NVRTC (csrc/runtime/jit.cpp), one module per parameter
// setting, after a generated prefix #defines the setting (CST_TBX ... CST_PF) and the
// stencil (CST_KIND, CST_R).  This is csTuner's "code generation writes the sampled
// parameter settings into CUDA kernels", done B200-first: every knob of
// Table I is a compile-time constant here.
//
// Paths:
//   fast streaming path   use_streaming=2, T_SD = TB_SD*BM_SD*CM_SD = 1 (2.5-D blocking,
//                         P:63): a register queue (gather) or 2r+1 rotating accumulators
//                         (retiming) along the streamed axis; in-plane operands from
//                         a TMA/mbarrier ring (staging 3), an ld/st smem ring with register
//                         prefetch (staging 2) or L1/L2 (staging 1).
//   generic streaming     T_SD > 1: ring of D*T_SD + 2r planes, gather from smem.
//   3-D tile path         use_streaming=1: (T+2r)^3 box in smem (TMA or ld/st) or L1/L2.
// Concurrent streaming (SB) splits the streamed axis into chunks = gridDim.y.
// Merging: thread t owns, per dim, points  c*(TB*BM) + t*BM + b  (b < BM, c < CM).
#include "cst_params.h"
#include "cst_ptx.cuh"

// ------------------------------------------------------------------ configuration
constexpr int KIND = CST_KIND;  // 1 star, 2 box, 3 hypterm
constexpr int R = CST_R;
constexpr int TBX = CST_TBX, TBY = CST_TBY, TBZ = CST_TBZ;
constexpr int STAGING = CST_STAGING;  // 1 none, 2 smem ld/st, 3 TMA
constexpr int CONSTMEM = CST_CONST;   // 1 params, 2 __constant__
constexpr bool STREAM = CST_STREAM == 2;
constexpr int SD = CST_SD;  // 2 y, 3 z (streaming); 1 when off
constexpr int SB = CST_SB;
constexpr int UFX = CST_UFX, UFY = CST_UFY, UFZ = CST_UFZ;
constexpr int CMX = CST_CMX, CMY = CST_CMY, CMZ = CST_CMZ;
constexpr int BMX = CST_BMX, BMY = CST_BMY, BMZ = CST_BMZ;
constexpr bool RETIME = CST_RET == 2;
constexpr int PF = CST_PF;  // pipeline stages (1 = no prefetch)

constexpr int NIN = KIND == 3 ? 8 : 1;
constexpr int NOUT = KIND == 3 ? 5 : 1;
constexpr int NTHR = TBX * TBY * TBZ;
constexpr int TX = TBX * BMX * CMX, TY = TBY * BMY * CMY, TZ = TBZ * BMZ * CMZ;

// streaming-axis view: a = x, b = the other in-plane dim, s = streamed dim
constexpr bool SZ = (SD == 3);
constexpr int TBA = TBX, TBB = SZ ? TBY : TBZ, TBS = SZ ? TBZ : TBY;
constexpr int BMA = BMX, BMB = SZ ? BMY : BMZ, BMS = SZ ? BMZ : BMY;
constexpr int CMA = CMX, CMB = SZ ? CMY : CMZ, CMS = SZ ? CMZ : CMY;
constexpr int UFA = UFX, UFB = SZ ? UFY : UFZ, UFS = SZ ? UFZ : UFY;
constexpr int TA = TBA * BMA * CMA, TB = TBB * BMB * CMB, TS = TBS * BMS * CMS;

__constant__ double c_coef[CST_MAX_COEF];

struct Ctx {
  const cst_kparams& P;
  __device__ __forceinline__ double coef(int i) const {
    if constexpr (CONSTMEM == 2) return c_coef[i];
    else return P.coef[i];
  }
};

__device__ __forceinline__ int merged_pos(int i, int t, int TBd, int BMd) {
  // i-th point (0 <= i < BM*CM) of thread t along one dim (block + cyclic merging)
  return (i / BMd) * (TBd * BMd) + t * BMd + (i % BMd);
}

// star coefficient index of offset k (k != 0) along axis (0 x, 1 y, 2 z)
__host__ __device__ constexpr int star_ci(int axis, int k) {
  return 1 + axis * 2 * R + (k < 0 ? k + R : k + R - 1);
}
constexpr int AX_A = 0, AX_B = SZ ? 1 : 2, AX_S = SZ ? 2 : 1;

// =============================================================================
// Point definitions over an accessor U(array, dx, dy, dz) — same terms as the oracle
// (DESIGN.md §2); fma contraction and the retimed orders are the only differences.
// =============================================================================
template <class Acc>
__device__ __forceinline__ void star_point(const Ctx& C, const Acc& U, double* o) {
  double s;
  if constexpr (!RETIME) {
    s = C.coef(0) * U(0, 0, 0, 0);
#pragma unroll
    for (int axis = 0; axis < 3; ++axis)
#pragma unroll
      for (int k = -R; k <= R; ++k) {
        if (k == 0) continue;
        s = fma(C.coef(star_ci(axis, k)),
                U(0, axis == 0 ? k : 0, axis == 1 ? k : 0, axis == 2 ? k : 0), s);
      }
  } else {
    // retimed order: by plane along the streamed axis (z when not streaming)
    constexpr int AS = STREAM ? AX_S : 2;
    constexpr int A1 = 0, A2 = (AS == 2) ? 1 : 2;
    s = 0.0;
#pragma unroll
    for (int k = -R; k <= R; ++k) {
      if (k == 0) {
        double ip = C.coef(0) * U(0, 0, 0, 0);
#pragma unroll
        for (int kk = -R; kk <= R; ++kk) {
          if (kk == 0) continue;
          ip = fma(C.coef(star_ci(A1, kk)), U(0, kk, 0, 0), ip);
        }
#pragma unroll
        for (int kk = -R; kk <= R; ++kk) {
          if (kk == 0) continue;
          ip = fma(C.coef(star_ci(A2, kk)), U(0, 0, A2 == 1 ? kk : 0, A2 == 2 ? kk : 0), ip);
        }
        s += ip;
      } else {
        s = fma(C.coef(star_ci(AS, k)), U(0, 0, AS == 1 ? k : 0, AS == 2 ? k : 0), s);
      }
    }
  }
  o[0] = s;
}

template <class Acc>
__device__ __forceinline__ void box_point(const Ctx& C, const Acc& U, double* o) {
  constexpr int W = 2 * R + 1;
  double s = 0.0;
  if constexpr (!RETIME || !STREAM || SZ) {
#pragma unroll
    for (int dz = -R; dz <= R; ++dz)
#pragma unroll
      for (int dy = -R; dy <= R; ++dy)
#pragma unroll
        for (int dx = -R; dx <= R; ++dx)
          s = fma(C.coef(((dz + R) * W + (dy + R)) * W + (dx + R)), U(0, dx, dy, dz), s);
  } else {
    // retimed, streaming along y: by plane along y
#pragma unroll
    for (int dy = -R; dy <= R; ++dy)
#pragma unroll
      for (int dz = -R; dz <= R; ++dz)
#pragma unroll
        for (int dx = -R; dx <= R; ++dx)
          s = fma(C.coef(((dz + R) * W + (dy + R)) * W + (dx + R)), U(0, dx, dy, dz), s);
  }
  o[0] = s;
}

// Hypterm-like (Table III "hypterm"): inputs cons1..4 = 0..3, q1..4 = 4..7.
template <class Acc>
__device__ __forceinline__ void hypterm_point(const Ctx& C, const Acc& U, double* flux) {
#pragma unroll
  for (int d = 0; d < 3; ++d) {
    const double dxi = C.coef(4 + d);
    double t[5];
#pragma unroll
    for (int f = 0; f < 5; ++f) {
      double sum = 0.0;
#pragma unroll
      for (int k = 1; k <= 4; ++k) {
        auto at = [&](int arr, int kk) {
          return U(arr, d == 0 ? kk : 0, d == 1 ? kk : 0, d == 2 ? kk : 0);
        };
        const int qd = 4 + d;
        double e;
        if (f == 0) {
          e = at(d, k) - at(d, -k);
        } else if (f <= 3) {
          const int cm = f - 1;
          e = fma(at(cm, k), at(qd, k), -(at(cm, -k) * at(qd, -k)));
          if (f - 1 == d) e = e + (at(7, k) - at(7, -k));
        } else {
          e = fma(at(3, k), at(qd, k), -(at(3, -k) * at(qd, -k))) +
              fma(at(7, k), at(qd, k), -(at(7, -k) * at(qd, -k)));
        }
        sum = (k == 1) ? C.coef(k - 1) * e : fma(C.coef(k - 1), e, sum);
      }
      t[f] = dxi * sum;
    }
#pragma unroll
    for (int f = 0; f < 5; ++f) flux[f] = (d == 0) ? -t[f] : flux[f] - t[f];
  }
}

template <class Acc>
__device__ __forceinline__ void point(const Ctx& C, const Acc& U, double* o) {
  if constexpr (KIND == 1) star_point(C, U, o);
  else if constexpr (KIND == 2) box_point(C, U, o);
  else hypterm_point(C, U, o);
}

// =============================================================================
// shared helpers
// =============================================================================
__device__ __forceinline__ int thread_x() { return (int)(threadIdx.x % TBX); }
__device__ __forceinline__ int thread_y() { return (int)((threadIdx.x / TBX) % TBY); }
__device__ __forceinline__ int thread_z() { return (int)(threadIdx.x / (TBX * TBY)); }

__host__ __device__ constexpr int round_slot(int elems) { return ((elems * 8 + 127) / 128) * 128 / 8; }

// =============================================================================
// 3-D tile path (use_streaming = 1)
// =============================================================================
__device__ __forceinline__ void kernel_tile3d(const cst_kparams& P, double* smem) {
  Ctx C{P};
  constexpr int BX = TX + 2 * R, BY = TY + 2 * R, BZ = TZ + 2 * R;
  constexpr int BOX = BX * BY * BZ;
  constexpr int BOXS = round_slot(BOX);
  const int tile_xy = blockIdx.x;
  const int x0 = (tile_xy % P.tiles_a) * TX;
  const int y0 = (tile_xy / P.tiles_a) * TY;
  const int z0 = blockIdx.y * TZ;
  const int tx = thread_x(), ty = thread_y(), tz = thread_z();
  const int tid = threadIdx.x;

  if constexpr (STAGING == 3) {
    u64* bar = (u64*)(smem + NIN * BOXS);
    if (tid == 0) {
      mbar_init(bar, 1);
      fence_mbar_init();
    }
    __syncthreads();
    if (tid == 0) {
      mbar_arrive_expect_tx(bar, NIN * BOX * 8);
#pragma unroll
      for (int a = 0; a < NIN; ++a)
        tma_load_3d(smem + a * BOXS, &P.tma[a], bar, P.tox + x0 - R, P.toy + y0 - R,
                    P.toz + z0 - R);
    }
    mbar_wait(bar, 0);
  } else if constexpr (STAGING == 2) {
    for (int e = tid; e < NIN * BOX; e += NTHR) {
      const int a = e / BOX, r = e % BOX;
      const int ex = r % BX, ey = (r / BX) % BY, ez = r / (BX * BY);
      const int gx = x0 - R + ex, gy = y0 - R + ey, gz = z0 - R + ez;
      double v = 0.0;
      if (gx < P.nx + R && gy < P.ny + R && gz < P.nz + R)
        v = P.in[a][gx + gy * P.py + gz * P.pz];
      smem[a * BOXS + r] = v;
    }
    __syncthreads();
  }

#pragma unroll(UFZ)
  for (int iz = 0; iz < BMZ * CMZ; ++iz) {
    const int lz = merged_pos(iz, tz, TBZ, BMZ);
#pragma unroll(UFY)
    for (int iy = 0; iy < BMY * CMY; ++iy) {
      const int ly = merged_pos(iy, ty, TBY, BMY);
#pragma unroll(UFX)
      for (int ix = 0; ix < BMX * CMX; ++ix) {
        const int lx = merged_pos(ix, tx, TBX, BMX);
        const int x = x0 + lx, y = y0 + ly, z = z0 + lz;
        if (x >= P.nx || y >= P.ny || z >= P.nz) continue;
        double o[NOUT];
        if constexpr (STAGING == 1) {
          const long long off = x + y * P.py + z * P.pz;
          auto U = [&](int a, int dx, int dy, int dz) {
            return ldg_nc(P.in[a] + off + dx + dy * P.py + dz * P.pz);
          };
          point(C, U, o);
        } else {
          auto U = [&](int a, int dx, int dy, int dz) {
            return smem[a * BOXS + ((lz + R + dz) * BY + (ly + R + dy)) * BX + lx + R + dx];
          };
          point(C, U, o);
        }
        const long long off = x + y * P.py + z * P.pz;
#pragma unroll
        for (int q = 0; q < NOUT; ++q) P.out[q][off] = o[q];
      }
    }
  }
}

// =============================================================================
// streaming geometry shared by both streaming paths
// =============================================================================
struct SGeo {
  int n_a, n_b, n_s;
  long long st_b, st_s;  // element strides of b and s
  int a0, b0, s_start, s_end;
};

__device__ __forceinline__ SGeo stream_geo(const cst_kparams& P) {
  SGeo g;
  g.n_a = P.nx;
  g.n_b = SZ ? P.ny : P.nz;
  g.n_s = SZ ? P.nz : P.ny;
  g.st_b = SZ ? P.py : P.pz;
  g.st_s = SZ ? P.pz : P.py;
  const int tile = blockIdx.x;
  g.a0 = (tile % P.tiles_a) * TA;
  g.b0 = (tile / P.tiles_a) * TB;
  g.s_start = blockIdx.y * SB;
  g.s_end = min(g.n_s, g.s_start + SB);
  return g;
}

// TMA coordinates of in-plane box origin (a0-R, b0-R) at stream plane p
__device__ __forceinline__ void tma_plane(const cst_kparams& P, const SGeo& g, double* dst,
                                          u64* bar, int p) {
#pragma unroll
  for (int a = 0; a < NIN; ++a) {
    constexpr int PA = TA + 2 * R, PB = TB + 2 * R;
    constexpr int SLOT = round_slot(PA * PB);
    if constexpr (SZ)
      tma_load_3d(dst + a * SLOT, &P.tma[a], bar, P.tox + g.a0 - R, P.toy + g.b0 - R,
                  P.toz + p);
    else
      tma_load_3d(dst + a * SLOT, &P.tma[a], bar, P.tox + g.a0 - R, P.toy + p,
                  P.toz + g.b0 - R);
  }
}

// cooperative ld/st copy of one plane (all arrays) into a ring slot
template <int PA, int PB, int SLOT>
__device__ __forceinline__ void ldst_plane(const cst_kparams& P, const SGeo& g, double* dst,
                                           int p) {
  constexpr int PL = PA * PB;
  for (int e = threadIdx.x; e < NIN * PL; e += NTHR) {
    const int a = e / PL, r = e % PL;
    const int ea = r % PA, eb = r / PA;
    const int ga = g.a0 - R + ea, gb = g.b0 - R + eb;
    double v = 0.0;
    if (ga < g.n_a + R && gb < g.n_b + R) v = P.in[a][ga + gb * g.st_b + p * g.st_s];
    dst[a * SLOT + r] = v;
  }
}

// =============================================================================
// fast streaming path, T_SD == 1: star
// =============================================================================
__device__ __forceinline__ void kernel_star_stream1(const cst_kparams& P, double* smem) {
  Ctx C{P};
  constexpr int PA = TA + 2 * R, PB = TB + 2 * R;
  constexpr int PL = PA * PB;
  constexpr int SLOT = round_slot(PL);
  constexpr int D = PF;
  constexpr int NP = STAGING == 1 ? 1 : D + (RETIME ? 0 : R);
  constexpr int NCA = BMA * CMA, NCB = BMB * CMB, NC = NCA * NCB;
  constexpr int W = 2 * R + 1;
  constexpr int FR = (NIN * PL + NTHR - 1) / NTHR;  // ld/st prefetch fragment per thread

  const SGeo g = stream_geo(P);
  const int ta = thread_x();
  const int tb = SZ ? thread_y() : thread_z();
  const int tid = threadIdx.x;
  const int n_planes = (g.s_end - g.s_start) + 2 * R;
  const double* __restrict__ in = P.in[0];
  double* __restrict__ out = P.out[0];
  u64* bars = (u64*)(smem + NP * SLOT);

  int la[NC], lb[NC];
  bool ok[NC];
#pragma unroll
  for (int i = 0; i < NC; ++i) {
    la[i] = merged_pos(i % NCA, ta, TBA, BMA);
    lb[i] = merged_pos(i / NCA, tb, TBB, BMB);
    ok[i] = (g.a0 + la[i] < g.n_a) && (g.b0 + lb[i] < g.n_b);
  }
  const long long col0 = (long long)g.a0 + (long long)g.b0 * g.st_b;

  double acc[NC][W];  // retimed: acc[i][m] = output plane p-R+m ; gather: queue of centres
#pragma unroll
  for (int i = 0; i < NC; ++i)
#pragma unroll
    for (int m = 0; m < W; ++m) acc[i][m] = 0.0;

  double frag[D > 1 && STAGING == 2 ? (D - 1) * FR : 1];

  // ---- prologue: first D planes in flight
  if constexpr (STAGING == 3) {
    if (tid == 0) {
      for (int s = 0; s < NP; ++s) mbar_init(&bars[s], 1);
      fence_mbar_init();
    }
    __syncthreads();
    if (tid == 0) {
      for (int j = 0; j < D && j < n_planes; ++j) {
        mbar_arrive_expect_tx(&bars[j % NP], NIN * PL * 8);
        tma_plane(P, g, smem + (j % NP) * NIN * SLOT, &bars[j % NP], g.s_start - R + j);
      }
    }
  } else if constexpr (STAGING == 2) {
    ldst_plane<PA, PB, SLOT>(P, g, smem, g.s_start - R);
    if constexpr (D > 1) {
#pragma unroll
      for (int f = 0; f < D - 1; ++f) {
        const int p = g.s_start - R + 1 + f;
#pragma unroll
        for (int q = 0; q < FR; ++q) {
          const int e = tid + q * NTHR;
          double v = 0.0;
          if (e < NIN * PL && 1 + f < n_planes) {
            const int r = e % PL;
            const int ga = g.a0 - R + r % PA, gb = g.b0 - R + r / PA;
            if (ga < g.n_a + R && gb < g.n_b + R) v = in[ga + gb * g.st_b + (long long)p * g.st_s];
          }
          frag[f * FR + q] = v;
        }
      }
    }
    __syncthreads();
  }

  // in-plane accessor of plane held in ring slot `slot` (or global plane p)
  auto inplane = [&](int i, int slot, int p) -> double {
    // c0*u + sum_a + sum_b ; summation order c0, a(=x), b
    if constexpr (STAGING == 1) {
      const double* c = in + col0 + la[i] + (long long)lb[i] * g.st_b + (long long)p * g.st_s;
      double s = C.coef(0) * ldg_nc(c);
#pragma unroll
      for (int k = -R; k <= R; ++k)
        if (k != 0) s = fma(C.coef(star_ci(AX_A, k)), ldg_nc(c + k), s);
#pragma unroll
      for (int k = -R; k <= R; ++k)
        if (k != 0) s = fma(C.coef(star_ci(AX_B, k)), ldg_nc(c + k * g.st_b), s);
      return s;
    } else {
      const double* c = smem + slot * NIN * SLOT + (lb[i] + R) * PA + la[i] + R;
      double s = C.coef(0) * c[0];
#pragma unroll
      for (int k = -R; k <= R; ++k)
        if (k != 0) s = fma(C.coef(star_ci(AX_A, k)), c[k], s);
#pragma unroll
      for (int k = -R; k <= R; ++k)
        if (k != 0) s = fma(C.coef(star_ci(AX_B, k)), c[k * PA], s);
      return s;
    }
  };
  auto centre = [&](int i, int slot, int p) -> double {
    if constexpr (STAGING == 1)
      return ldg_nc(in + col0 + la[i] + (long long)lb[i] * g.st_b + (long long)p * g.st_s);
    else
      return smem[slot * NIN * SLOT + (lb[i] + R) * PA + la[i] + R];
  };

#pragma unroll(UFS)
  for (int j = 0; j < n_planes; ++j) {
    const int p = g.s_start - R + j;
    const int slot = j % NP;
    if constexpr (STAGING == 3) mbar_wait(&bars[slot], (u32)((j / NP) & 1));

    if constexpr (RETIME) {
      // retiming: plane p contributes ws[p-o]*u to outputs o = p-R..p+R and its
      // in-plane partial sum to output p; output p-R is complete afterwards.
#pragma unroll
      for (int i = 0; i < NC; ++i) {
        const double v = centre(i, slot, p);
#pragma unroll
        for (int m = 0; m < W; ++m) {
          if (m == R) continue;
          acc[i][m] = fma(C.coef(star_ci(AX_S, R - m)), v, acc[i][m]);
        }
        acc[i][R] += inplane(i, slot, p);
      }
      if (j >= 2 * R) {
        const long long so = (long long)(p - R) * g.st_s;
#pragma unroll
        for (int i = 0; i < NC; ++i)
          if (ok[i]) out[col0 + la[i] + (long long)lb[i] * g.st_b + so] = acc[i][0];
      }
#pragma unroll
      for (int i = 0; i < NC; ++i) {
#pragma unroll
        for (int m = 0; m < W - 1; ++m) acc[i][m] = acc[i][m + 1];
        acc[i][W - 1] = 0.0;
      }
    } else {
      // gather: register queue of the 2R+1 centre values along s (2.5-D blocking)
#pragma unroll
      for (int i = 0; i < NC; ++i) {
#pragma unroll
        for (int m = 0; m < W - 1; ++m) acc[i][m] = acc[i][m + 1];
        acc[i][W - 1] = centre(i, slot, p);
      }
      if (j >= 2 * R) {
        const int po = p - R;
        const int slot_o = (j - R) % NP;
        const long long so = (long long)po * g.st_s;
#pragma unroll
        for (int i = 0; i < NC; ++i) {
          double s = inplane(i, slot_o, po);
#pragma unroll
          for (int k = -R; k <= R; ++k)
            if (k != 0) s = fma(C.coef(star_ci(AX_S, k)), acc[i][R + k], s);
          if (ok[i]) out[col0 + la[i] + (long long)lb[i] * g.st_b + so] = s;
        }
      }
    }

    // ---- release the oldest live slot and refill it with plane j + D
    if constexpr (STAGING == 3) {
      __syncthreads();
      if (tid == 0 && j + D < n_planes) {
        const int sl = (j + D) % NP;
        fence_proxy_async();
        mbar_arrive_expect_tx(&bars[sl], NIN * PL * 8);
        tma_plane(P, g, smem + sl * NIN * SLOT, &bars[sl], p + D);
      }
    } else if constexpr (STAGING == 2) {
      __syncthreads();
      if (j + 1 < n_planes) {
        double* dst = smem + ((j + 1) % NP) * NIN * SLOT;
        if constexpr (D == 1) {
          ldst_plane<PA, PB, SLOT>(P, g, dst, p + 1);
        } else {
#pragma unroll
          for (int q = 0; q < FR; ++q) {
            const int e = tid + q * NTHR;
            if (e < NIN * PL) dst[e] = frag[q];
          }
#pragma unroll
          for (int f = 0; f < D - 2; ++f)
#pragma unroll
            for (int q = 0; q < FR; ++q) frag[f * FR + q] = frag[(f + 1) * FR + q];
          const int pn = p + D;
#pragma unroll
          for (int q = 0; q < FR; ++q) {
            const int e = tid + q * NTHR;
            double v = 0.0;
            if (e < NIN * PL && j + D < n_planes) {
              const int r = e % PL;
              const int ga = g.a0 - R + r % PA, gb = g.b0 - R + r / PA;
              if (ga < g.n_a + R && gb < g.n_b + R)
                v = in[ga + gb * g.st_b + (long long)pn * g.st_s];
            }
            frag[(D - 2) * FR + q] = v;
          }
        }
      }
      __syncthreads();
    }
  }
}

// =============================================================================
// generic streaming path (any kind, any T_SD): ring of D*TS + 2R planes, gather
// =============================================================================
__device__ __forceinline__ void kernel_stream_generic(const cst_kparams& P, double* smem) {
  Ctx C{P};
  constexpr int PA = TA + 2 * R, PB = TB + 2 * R;
  constexpr int PL = PA * PB;
  constexpr int SLOT = round_slot(PL);
  constexpr int D = PF;
  constexpr int NP = D * TS + 2 * R;
  const SGeo g = stream_geo(P);
  const int ta = thread_x();
  const int tb = SZ ? thread_y() : thread_z();
  const int ts = SZ ? thread_z() : thread_y();
  const int tid = threadIdx.x;
  const int n_out = g.s_end - g.s_start;
  const int n_planes = n_out + 2 * R;
  const int steps = (n_out + TS - 1) / TS;
  u64* bars = (u64*)(smem + NP * NIN * SLOT);

  auto issue = [&](int j) {  // load plane j (sequence index) into its slot
    if (j >= n_planes) return;
    const int sl = j % NP;
    if constexpr (STAGING == 3) {
      if (tid == 0) {
        fence_proxy_async();
        mbar_arrive_expect_tx(&bars[sl], NIN * PL * 8);
        tma_plane(P, g, smem + sl * NIN * SLOT, &bars[sl], g.s_start - R + j);
      }
    } else if constexpr (STAGING == 2) {
      ldst_plane<PA, PB, SLOT>(P, g, smem + sl * NIN * SLOT, g.s_start - R + j);
    }
  };

  if constexpr (STAGING == 3) {
    if (tid == 0) {
      for (int s = 0; s < NP; ++s) mbar_init(&bars[s], 1);
      fence_mbar_init();
    }
    __syncthreads();
  }
  if constexpr (STAGING >= 2) {
    for (int j = 0; j < NP; ++j) issue(j);
    if constexpr (STAGING == 2) __syncthreads();
  }

  for (int k = 0; k < steps; ++k) {
    if constexpr (STAGING == 3) {
      const int jhi = min(n_planes, (k + 1) * TS + 2 * R);
      for (int j = k * TS; j < jhi; ++j) mbar_wait(&bars[j % NP], (u32)((j / NP) & 1));
    }
#pragma unroll(UFS)
    for (int is = 0; is < BMS * CMS; ++is) {
      const int ls = merged_pos(is, ts, TBS, BMS);
      const int s = g.s_start + k * TS + ls;
#pragma unroll(UFB)
      for (int ib = 0; ib < BMB * CMB; ++ib) {
        const int lb = merged_pos(ib, tb, TBB, BMB);
#pragma unroll(UFA)
        for (int ia = 0; ia < BMA * CMA; ++ia) {
          const int la = merged_pos(ia, ta, TBA, BMA);
          const int a = g.a0 + la, b = g.b0 + lb;
          if (a >= g.n_a || b >= g.n_b || s >= g.s_end) continue;
          const long long off = a + b * g.st_b + (long long)s * g.st_s;
          double o[NOUT];
          if constexpr (STAGING == 1) {
            auto U = [&](int arr, int dx, int dy, int dz) {
              return ldg_nc(P.in[arr] + off + dx + dy * P.py + dz * P.pz);
            };
            point(C, U, o);
          } else {
            const int jp = s - g.s_start + R;  // sequence index of the point's plane
            auto U = [&](int arr, int dx, int dy, int dz) {
              const int da = dx, db = SZ ? dy : dz, ds = SZ ? dz : dy;
              return smem[((jp + ds) % NP) * NIN * SLOT + arr * SLOT + (lb + R + db) * PA +
                          la + R + da];
            };
            point(C, U, o);
          }
#pragma unroll
          for (int q = 0; q < NOUT; ++q) P.out[q][off] = o[q];
        }
      }
    }
    if constexpr (STAGING >= 2) {
      __syncthreads();
      for (int j = (k + D) * TS + 2 * R; j < (k + D + 1) * TS + 2 * R; ++j) issue(j);
      if constexpr (STAGING == 2) __syncthreads();
    }
  }
}

// =============================================================================
// entry point
// =============================================================================
extern "C" __global__ void __launch_bounds__(NTHR) cst_kernel(const __grid_constant__ cst_kparams P) {
  extern __shared__ __align__(128) double cst_smem[];
  if constexpr (!STREAM) {
    kernel_tile3d(P, cst_smem);
  } else if constexpr (KIND == 1 && TS == 1) {
    kernel_star_stream1(P, cst_smem);
  } else {
    kernel_stream_generic(P, cst_smem);
  }
}
