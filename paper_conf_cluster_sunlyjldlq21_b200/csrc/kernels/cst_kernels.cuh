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

#ifndef CST_EMPTY_BARRIERS
#define CST_EMPTY_BARRIERS 0
#endif
#ifndef CST_HYP_SCALAR
#define CST_HYP_SCALAR 0
#endif
#ifndef CST_REMOTE
#define CST_REMOTE 0  // 1: fused-halo twin (z-slab boundary launches, NEXT-3)
#endif
#ifndef CST_QSTORE
#define CST_QSTORE 1  // streamed-direction state: 1 registers, 2 tensor memory (TMEM)
#endif
#ifndef CST_HYP_ROWS
#define CST_HYP_ROWS 1  // TMEM hypterm: in-plane terms by row streaming
#endif

// ------------------------------------------------------------------ configuration
constexpr int KIND = CST_KIND;  // 1 star, 2 box, 3 hypterm, 4 rhs4center-like
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
constexpr bool QTM = CST_QSTORE == 2;

constexpr int NIN = KIND == 3 ? 8 : (KIND == 4 ? 5 : 1);
constexpr int NOUT = KIND == 3 ? 5 : (KIND == 4 ? 3 : 1);
constexpr int NTHR = TBX * TBY * TBZ;
constexpr int TX = TBX * BMX * CMX, TY = TBY * BMY * CMY, TZ = TBZ * BMZ * CMZ;

// streaming-axis view: a = x, b = the other in-plane dim, s = streamed dim
constexpr bool SZ = (SD == 3);
constexpr int TBA = TBX, TBB = SZ ? TBY : TBZ, TBS = SZ ? TBZ : TBY;
constexpr int BMA = BMX, BMB = SZ ? BMY : BMZ, BMS = SZ ? BMZ : BMY;
constexpr int CMA = CMX, CMB = SZ ? CMY : CMZ, CMS = SZ ? CMZ : CMY;
constexpr int UFA = UFX, UFB = SZ ? UFY : UFZ, UFS = SZ ? UFZ : UFY;
constexpr int TA = TBA * BMA * CMA, TB = TBB * BMB * CMB, TS = TBS * BMS * CMS;
// minimum resident CTAs requested from ptxas (__launch_bounds__); 3 would fit the
// 45-accumulator hypterm path in 168 registers but spills a few bytes, so it stays 0
// (= no request, ptxas' own heuristic, which measured best)
constexpr int MINB = 0;

__constant__ double c_coef[CST_MAX_COEF];

struct Ctx {
  const cst_kparams& P;
  __device__ __forceinline__ double coef(int i) const {
    if constexpr (CONSTMEM == 2) return c_coef[i];
    else return P.coef[i];
  }
};

// Store one interior output value.  In a z-slab boundary launch of the fused halo
// exchange the same value is also stored into the neighbour rank's
// halo through its peer-mapped buffer (NVLink / NVSwitch): rout[q] is offset so that the
// launch's own element offset addresses the neighbour's matching halo element.  A
// compile-time twin (CST_REMOTE): the plain variant carries no trace of it.
__device__ __forceinline__ void put(const cst_kparams& P, int q, long long off, double v) {
  P.out[q][off] = v;
  if constexpr (CST_REMOTE) P.rout[q][off] = v;
}

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

// rhs4center-like (NEXT-1; Table III "rhs4center"): inputs u1, u2, u3, mu, lambda,
// outputs r1..r3, coefficients [s_x, s_y, s_z]; the oracle's terms in the oracle's order,
//   r_i = sum_d s_d^2 V_d[mu + delta_id (mu + la)](u_i)
//       + sum_{d != i} s_d s_i (D_d[mu D_i u_d] + D_i[la D_d u_d]),
// with the constant factors folded (host-precomputed in the coefficient bank):
// kcoef[3 + d] = s_d^2 / 6 scales the unscaled V sum, kcoef[6 + pair(d, i)] = s_d s_i / 144
// scales the unscaled outer(inner) difference of each mixed term.
// Two x-adjacent points evaluated in lockstep (the paired rhs4 path): the same operations
// in the same order per lane as the scalar code.
struct dpair {
  double x, y;
};
__device__ __forceinline__ dpair operator+(dpair a, dpair b) { return {a.x + b.x, a.y + b.y}; }
__device__ __forceinline__ dpair operator-(dpair a, dpair b) { return {a.x - b.x, a.y - b.y}; }
__device__ __forceinline__ dpair operator*(dpair a, dpair b) { return {a.x * b.x, a.y * b.y}; }
__device__ __forceinline__ dpair operator*(double a, dpair b) { return {a * b.x, a * b.y}; }
__device__ __forceinline__ dpair fma(double a, dpair b, dpair c) {
  return {fma(a, b.x, c.x), fma(a, b.y, c.y)};
}
__device__ __forceinline__ dpair fma(dpair a, dpair b, dpair c) {
  return {fma(a.x, b.x, c.x), fma(a.y, b.y, c.y)};
}

template <class T, class Acc>
__device__ __forceinline__ void rhs4_point_t(const Ctx& C, const Acc& U, T* r) {
  auto at = [&](int arr, int d, int k, int d2, int k2) {
    int o[3] = {0, 0, 0};
    o[d] += k;
    o[d2] += k2;
    return U(arr, o[0], o[1], o[2]);
  };
#pragma unroll
  for (int i = 0; i < 3; ++i) {
    T acc{};
#pragma unroll
    for (int d = 0; d < 3; ++d) {
      auto a = [&](int k) {
        const T m = at(3, d, k, d, 0);
        return d == i ? fma(2.0, m, at(4, d, k, d, 0)) : m;
      };
      auto f = [&](int k) { return at(i, d, k, d, 0); };
      const T am2 = a(-2), am1 = a(-1), a0 = a(0), ap1 = a(1), ap2 = a(2);
      const T m1 = fma(-0.75, a0 + am2, am1);
      const T m2 = fma(3.0, a0 + am1, am2 + ap1);
      const T m3 = fma(3.0, ap1 + a0, am1 + ap2);
      const T m4 = fma(-0.75, a0 + ap2, ap1);
      const T f0 = f(0);
      T v = m1 * (f(-2) - f0);
      v = fma(m2, f(-1) - f0, v);
      v = fma(m3, f(1) - f0, v);
      v = fma(m4, f(2) - f0, v);
      acc = d == 0 ? C.coef(3 + d) * v : fma(C.coef(3 + d), v, acc);
    }
#pragma unroll
    for (int d = 0; d < 3; ++d) {
      if (d == i) continue;
      auto mixed = [&](int outer, int inner, int coef, int comp) {
        auto inner_d = [&](int ko) {
          const T g = fma(8.0, at(comp, outer, ko, inner, 1) - at(comp, outer, ko, inner, -1),
                               at(comp, outer, ko, inner, -2) - at(comp, outer, ko, inner, 2));
          return at(coef, outer, ko, outer, 0) * g;
        };
        return fma(8.0, inner_d(1) - inner_d(-1), inner_d(-2) - inner_d(2));
      };
      const double w = C.coef(6 + (d + i - 1));  // pair (0,1) -> 6, (0,2) -> 7, (1,2) -> 8
      acc = fma(w, mixed(d, i, 3, d), acc);
      acc = fma(w, mixed(i, d, 4, d), acc);
    }
    r[i] = acc;
  }
}

template <class Acc>
__device__ __forceinline__ void rhs4_point(const Ctx& C, const Acc& U, double* r) {
  rhs4_point_t<double>(C, U, r);
}

template <class Acc>
__device__ __forceinline__ void point(const Ctx& C, const Acc& U, double* o) {
  if constexpr (KIND == 1) star_point(C, U, o);
  else if constexpr (KIND == 2) box_point(C, U, o);
  else if constexpr (KIND == 3) hypterm_point(C, U, o);
  else rhs4_point(C, U, o);
}

// =============================================================================
// shared helpers
// =============================================================================
__device__ __forceinline__ int thread_x() { return (int)(threadIdx.x % TBX); }
__device__ __forceinline__ int thread_y() { return (int)((threadIdx.x / TBX) % TBY); }
__device__ __forceinline__ int thread_z() { return (int)(threadIdx.x / (TBX * TBY)); }

__host__ __device__ constexpr int round_slot(int elems) { return ((elems * 8 + 127) / 128) * 128 / 8; }

// x-halo kept in shared memory / TMA boxes: R rounded up to even, so every box row starts
// 16-B aligned in global memory (TMA requirement) and double2 loads stay aligned.
constexpr int XR = R + (R & 1);

template <bool B, class T, class F>
struct Cond {
  using type = T;
};
template <class T, class F>
struct Cond<false, T, F> {
  using type = F;
};

template <int V>
struct IC {
  static constexpr int value = V;
};
template <int I, int N, class F>
__device__ __forceinline__ void static_for(F&& f) {
  if constexpr (I < N) {
    f(IC<I>{});
    static_for<I + 1, N>(f);
  }
}

// =============================================================================
// 3-D tile path (use_streaming = 1)
// =============================================================================
__device__ __forceinline__ void kernel_tile3d(const cst_kparams& P, double* smem) {
  Ctx C{P};
  constexpr int BX = TX + 2 * XR, BY = TY + 2 * R, BZ = TZ + 2 * R;
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
        tma_load_3d(smem + a * BOXS, &P.tma[a], bar, P.tox + x0 - XR, P.toy + y0 - R,
                    P.toz + z0 - R);
    }
    mbar_wait(bar, 0);
  } else if constexpr (STAGING == 2) {
    for (int e = tid; e < NIN * BOX; e += NTHR) {
      const int a = e / BOX, r = e % BOX;
      const int ex = r % BX, ey = (r / BX) % BY, ez = r / (BX * BY);
      const int gx = x0 - XR + ex, gy = y0 - R + ey, gz = z0 - R + ez;
      double v = 0.0;
      if (gx >= -R && gx < P.nx + R && gy < P.ny + R && gz < P.nz + R)
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
            return smem[a * BOXS + ((lz + R + dz) * BY + (ly + R + dy)) * BX + lx + XR + dx];
          };
          point(C, U, o);
        }
        const long long off = x + y * P.py + z * P.pz;
#pragma unroll
        for (int q = 0; q < NOUT; ++q) put(P, q, off, o[q]);
      }
    }
  }
}

// =============================================================================
// streaming geometry, plane staging (ring of plane slots; slot = NIN arrays)
// =============================================================================
constexpr int PA = TA + 2 * XR, PB = TB + 2 * R;
constexpr int PL = PA * PB;
constexpr int SLOT = round_slot(PL);

// Per-array halos of the hypterm TMA fast path (HTRIM): each input is staged with only the
// halos its terms read (Table III hypterm): cons1..4 and q4 enter the
// derivatives along every direction (a- and b-halos), q_a only along a, q_b only along b,
// q_s only through the streamed-direction products (no in-plane halo).  Every other path
// stages NIN uniform (PA x PB) slots; the layout functions then reduce to a * SLOT.
// Mirrored by the host (cst_api.cpp: TMA boxes; space.cpp: kernel_smem_bytes).
constexpr bool HTRIM = KIND == 3 && STAGING == 3 && STREAM && TS == 1 && CST_BT == 1;
constexpr int Q_A = 4, Q_B = SZ ? 5 : 6;  // q index of direction a (x) and b (y or z)
__host__ __device__ constexpr bool arr_halo_a(int a) { return !HTRIM || a < 4 || a == 7 || a == Q_A; }
__host__ __device__ constexpr bool arr_halo_b(int a) { return !HTRIM || a < 4 || a == 7 || a == Q_B; }
__host__ __device__ constexpr int arr_wa(int a) { return TA + (arr_halo_a(a) ? 2 * XR : 0); }
__host__ __device__ constexpr int arr_wb(int a) { return TB + (arr_halo_b(a) ? 2 * R : 0); }
__host__ __device__ constexpr int arr_off(int a) {
  int o = 0;
  for (int i = 0; i < a; ++i) o += round_slot(arr_wa(i) * arr_wb(i));
  return o;
}
__host__ __device__ constexpr int arr_txb(int n) {
  int b = 0;
  for (int i = 0; i < n; ++i) b += arr_wa(i) * arr_wb(i) * 8;
  return b;
}
constexpr int RSLOT = arr_off(NIN);      // elements of one ring slot (all arrays)
constexpr int TX_BYTES = arr_txb(NIN);   // TMA bytes of one plane (all arrays)
static_assert(HTRIM || (RSLOT == NIN * SLOT && TX_BYTES == NIN * PL * 8), "uniform layout");

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

// TMA: in-plane box origin (a0 - XR, b0 - R) at stream plane p, all arrays
__device__ __forceinline__ void tma_plane(const cst_kparams& P, const SGeo& g, double* dst,
                                          u64* bar, int p) {
#pragma unroll
  for (int a = 0; a < NIN; ++a) {
    const int oa = g.a0 - (arr_halo_a(a) ? XR : 0), ob = g.b0 - (arr_halo_b(a) ? R : 0);
    if constexpr (SZ)
      tma_load_3d(dst + arr_off(a), &P.tma[a], bar, P.tox + oa, P.toy + ob, P.toz + p);
    else
      tma_load_3d(dst + arr_off(a), &P.tma[a], bar, P.tox + oa, P.toy + p, P.toz + ob);
  }
}

// global value of element r (0 <= r < NIN*PL) of plane p, 0 outside the padded region
__device__ __forceinline__ double plane_elem(const cst_kparams& P, const SGeo& g, int e, int p) {
  const int a = e / PL, r = e % PL;
  const int ga = g.a0 - XR + r % PA, gb = g.b0 - R + r / PA;
  if (ga >= -R && ga < g.n_a + R && gb < g.n_b + R)
    return P.in[a][ga + gb * g.st_b + (long long)p * g.st_s];
  return 0.0;
}

__device__ __forceinline__ void ldst_plane(const cst_kparams& P, const SGeo& g, double* dst,
                                           int p) {
  for (int e = threadIdx.x; e < NIN * PL; e += NTHR) dst[(e / PL) * SLOT + e % PL] = plane_elem(P, g, e, p);
}

// plane accessors: element (la, lb) of the tile-local in-plane coordinates
struct SmemPlane {
  static constexpr bool VEC = true;
  const double* base;  // slot base of one array
  __device__ __forceinline__ double at(int la, int lb) const { return base[(lb + R) * PA + la + XR]; }
  __device__ __forceinline__ double2 at2(int la, int lb) const {
    return *reinterpret_cast<const double2*>(base + (lb + R) * PA + la + XR);
  }
};
// HTRIM slots: per-array pitch and origin (compile-time constants once the array loop is
// unrolled); a separate type so the uniform paths keep their one-pointer accessor
struct SmemPlaneV {
  static constexpr bool VEC = true;
  const double* base;
  int pitch;  // row pitch (elements)
  int org;    // element offset of tile point (0, 0)
  __device__ __forceinline__ double at(int la, int lb) const { return base[org + lb * pitch + la]; }
  __device__ __forceinline__ double2 at2(int la, int lb) const {
    return *reinterpret_cast<const double2*>(base + org + lb * pitch + la);
  }
};
using SPlane = typename Cond<HTRIM, SmemPlaneV, SmemPlane>::type;
// array a of the ring slot at `slot_base` (per-array layout; uniform unless HTRIM)
__device__ __forceinline__ SmemPlaneV splane_v(const double* slot_base, int a) {
  return SmemPlaneV{slot_base + arr_off(a), arr_wa(a),
                    (arr_halo_b(a) ? R : 0) * arr_wa(a) + (arr_halo_a(a) ? XR : 0)};
}
__device__ __forceinline__ SmemPlane splane_u(const double* slot_base, int a) {
  return SmemPlane{slot_base + arr_off(a)};
}
__device__ __forceinline__ auto splane(const double* slot_base, int a) {
  if constexpr (HTRIM) return splane_v(slot_base, a);
  else return splane_u(slot_base, a);
}
struct GlobPlane {
  static constexpr bool VEC = false;
  const double* base;  // &u(a0, b0, p)
  long long stb;
  __device__ __forceinline__ double at(int la, int lb) const { return ldg_nc(base + la + lb * stb); }
  __device__ __forceinline__ double2 at2(int la, int lb) const {
    return make_double2(at(la, lb), at(la + 1, lb));
  }
};

constexpr int NCA = BMA * CMA, NCB = BMB * CMB;
// rhs4 in the generic streaming path with BM_x = 2: two points per thread in lockstep
constexpr bool PAIRED = KIND == 4 && BMA == 2 && CMA == 1 && STAGING >= 2;
constexpr int W = 2 * R + 1;

// load the x-window [la0 - XR, la0 + BMA + XR) of row lb (only [la0-R, la0+BMA+R) used)
template <class LD>
__device__ __forceinline__ void load_xwin(const LD& ld, int la0, int lb, double* w) {
  constexpr int WX = BMA + 2 * XR;
  if constexpr (LD::VEC && (BMA % 2 == 0)) {
#pragma unroll
    for (int q = 0; q < WX / 2; ++q) {
      const double2 v = ld.at2(la0 - XR + 2 * q, lb);
      w[2 * q] = v.x;
      w[2 * q + 1] = v.y;
    }
  } else if constexpr (LD::VEC) {
    // odd run width: load the 16-B aligned superset with double2 (adjacent lanes then
    // share 16-B chunks -> broadcast) and select the lane's parity
    constexpr int NV = (WX + 2) / 2;
    const int odd = (la0 - XR) & 1;
    const int e0 = la0 - XR - odd;
    double raw[2 * NV];
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      const double2 v = ld.at2(e0 + 2 * q, lb);
      raw[2 * q] = v.x;
      raw[2 * q + 1] = v.y;
    }
#pragma unroll
    for (int q = 0; q < WX; ++q) w[q] = odd ? raw[q + 1] : raw[q];
  } else {
#pragma unroll
    for (int q = XR - R; q < WX - (XR - R); ++q) w[q] = ld.at(la0 - XR + q, lb);
  }
}

// =============================================================================
// star: in-plane part  ip = c0*u + sum_k wa[k] u(a+k) + sum_k wb[k] u(b+k)  (oracle order)
// register-blocked over the thread's BM_a x BM_b points (merging reuse)
// =============================================================================
template <class LD>
__device__ __forceinline__ void star_inplane(const Ctx& C, const LD& ld, const int* la,
                                             const int* lb, double (&ip)[NCB][NCA],
                                             double (&cen)[NCB][NCA]) {
#pragma unroll
  for (int ib = 0; ib < NCB; ++ib) {
#pragma unroll
    for (int ca = 0; ca < CMA; ++ca) {
      double w[BMA + 2 * XR];
      load_xwin(ld, la[ca * BMA], lb[ib], w);
#pragma unroll
      for (int b = 0; b < BMA; ++b) {
        const double c = w[XR + b];
        double s = C.coef(0) * c;
#pragma unroll
        for (int k = -R; k <= R; ++k)
          if (k != 0) s = fma(C.coef(star_ci(AX_A, k)), w[XR + b + k], s);
        ip[ib][ca * BMA + b] = s;
        cen[ib][ca * BMA + b] = c;
      }
    }
  }
#pragma unroll
  for (int cb = 0; cb < CMB; ++cb) {
    const int lb0 = lb[cb * BMB];
#pragma unroll
    for (int ia = 0; ia < NCA; ++ia) {
      constexpr bool PAIR = LD::VEC && (BMA % 2 == 0);
      if (PAIR && (ia % 2)) continue;
      double top[PAIR ? 2 : 1][R], bot[PAIR ? 2 : 1][R];
#pragma unroll
      for (int t = 0; t < R; ++t) {
        if constexpr (PAIR) {
          const double2 a = ld.at2(la[ia], lb0 - 1 - t);
          const double2 b = ld.at2(la[ia], lb0 + BMB + t);
          top[0][t] = a.x; top[1][t] = a.y;
          bot[0][t] = b.x; bot[1][t] = b.y;
        } else {
          top[0][t] = ld.at(la[ia], lb0 - 1 - t);
          bot[0][t] = ld.at(la[ia], lb0 + BMB + t);
        }
      }
#pragma unroll
      for (int pc = 0; pc < (PAIR ? 2 : 1); ++pc) {
        const int iac = ia + pc;
#pragma unroll
        for (int rb = 0; rb < BMB; ++rb) {
          double s = ip[cb * BMB + rb][iac];
#pragma unroll
          for (int k = -R; k <= R; ++k) {
            if (k == 0) continue;
            const int rr = rb + k;
            const double v = rr < 0 ? top[pc][-rr - 1]
                                    : (rr >= BMB ? bot[pc][rr - BMB] : cen[cb * BMB + rr][iac]);
            s = fma(C.coef(star_ci(AX_B, k)), v, s);
          }
          ip[cb * BMB + rb][iac] = s;
        }
      }
    }
  }
}

template <class LD>
__device__ __forceinline__ void load_centres(const LD& ld, const int* la, const int* lb,
                                             double (&cen)[NCB][NCA]) {
#pragma unroll
  for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
    for (int ia = 0; ia < NCA; ++ia) {
      if constexpr (LD::VEC && (BMA % 2 == 0)) {
        if (ia % 2) continue;
        const double2 v = ld.at2(la[ia], lb[ib]);
        cen[ib][ia] = v.x;
        cen[ib][ia + 1] = v.y;
      } else {
        cen[ib][ia] = ld.at(la[ia], lb[ib]);
      }
    }
}


// Retimed star plane update, fully in scatter form: every value loaded from plane p
// is added straight into the rotating accumulators — s-neighbours (2R per point), x-terms
// of its row and y-terms of the rows within R — so no per-point temporaries stay live.
// Logical accumulator m of a point = output plane p - R + m (phys (m + U) % W); the
// in-plane part belongs to m = R.
template <int U, class LD>
__device__ __forceinline__ void star_retimed_plane(const Ctx& C, const LD& ld, const int* la,
                                                   const int* lb,
                                                   double (&acc)[NCB][NCA][W]) {
  constexpr int MR = (R + U) % W;
#pragma unroll
  for (int cb = 0; cb < CMB; ++cb) {
    const int lb0 = lb[cb * BMB];
#pragma unroll
    for (int ca = 0; ca < CMA; ++ca) {
      const int la0 = la[ca * BMA];
#pragma unroll
      for (int wr = -R; wr < BMB + R; ++wr) {
        if (wr >= 0 && wr < BMB) {
          double w[BMA + 2 * XR];
          load_xwin(ld, la0, lb0 + wr, w);
#pragma unroll
          for (int b = 0; b < BMA; ++b) {
            double(&A)[W] = acc[cb * BMB + wr][ca * BMA + b];
            const double c = w[XR + b];
#pragma unroll
            for (int m = 0; m < W; ++m)  // s-direction scatter: plane p -> output p-R+m
              if (m != R) A[(m + U) % W] = fma(C.coef(star_ci(AX_S, R - m)), c, A[(m + U) % W]);
            double ip = C.coef(0) * c;
#pragma unroll
            for (int k = -R; k <= R; ++k)
              if (k != 0) ip = fma(C.coef(star_ci(AX_A, k)), w[XR + b + k], ip);
            A[MR] += ip;
#pragma unroll
            for (int rb = 0; rb < BMB; ++rb) {  // y-terms of the block rows
              const int k = wr - rb;
              if (k == 0 || k < -R || k > R) continue;
              double& B = acc[cb * BMB + rb][ca * BMA + b][MR];
              B = fma(C.coef(star_ci(AX_B, k)), c, B);
            }
          }
        } else {
          double v[BMA];
          if constexpr (LD::VEC && (BMA % 2 == 0)) {
#pragma unroll
            for (int b = 0; b < BMA; b += 2) {
              const double2 t = ld.at2(la0 + b, lb0 + wr);
              v[b] = t.x;
              v[b + 1] = t.y;
            }
          } else {
#pragma unroll
            for (int b = 0; b < BMA; ++b) v[b] = ld.at(la0 + b, lb0 + wr);
          }
#pragma unroll
          for (int b = 0; b < BMA; ++b)
#pragma unroll
            for (int rb = 0; rb < BMB; ++rb) {
              const int k = wr - rb;
              if (k < -R || k > R) continue;
              double& B = acc[cb * BMB + rb][ca * BMA + b][MR];
              B = fma(C.coef(star_ci(AX_B, k)), v[b], B);
            }
        }
      }
    }
  }
}

// =============================================================================
// box (r = 1): slice sums  S_ds(p) = sum_{db,da} c(ds, db, da) u(a+da, b+db, p)
// =============================================================================
__host__ __device__ constexpr int box_ci(int ds, int db, int da) {
  // coefficient c[dz][dy][dx] (z-major); s = z (SD = 3) or y (SD = 2)
  return SZ ? ((ds + R) * W + (db + R)) * W + (da + R) : ((db + R) * W + (ds + R)) * W + (da + R);
}

// accumulate slices ds = DS0 + q*DSTEP (q < NS) of plane `ld` into chains S[q][ib][ia]
// (db, da ascending within each chain)
template <int NS, int DS0, int DSTEP, class LD>
__device__ __forceinline__ void box_slices(const Ctx& C, const LD& ld, const int* la, const int* lb,
                                           double (&S)[NS][NCB][NCA]) {
#pragma unroll
  for (int cb = 0; cb < CMB; ++cb) {
    const int lb0 = lb[cb * BMB];
#pragma unroll
    for (int ca = 0; ca < CMA; ++ca) {
      const int la0 = la[ca * BMA];
#pragma unroll
      for (int wr = -R; wr < BMB + R; ++wr) {  // window rows
        double w[BMA + 2 * XR];
        load_xwin(ld, la0, lb0 + wr, w);
#pragma unroll
        for (int rb = 0; rb < BMB; ++rb) {
          const int db = wr - rb;
          if (db < -R || db > R) continue;
#pragma unroll
          for (int b = 0; b < BMA; ++b)
#pragma unroll
            for (int da = -R; da <= R; ++da)
#pragma unroll
              for (int q = 0; q < NS; ++q) {
                double& acc = S[q][cb * BMB + rb][ca * BMA + b];
                acc = fma(C.coef(box_ci(DS0 + q * DSTEP, db, da)), w[XR + b + da], acc);
              }
        }
      }
    }
  }
}

// =============================================================================
// fast streaming path, T_SD == 1 (star / box): one plane per step, rotation-unrolled
// =============================================================================
constexpr int RETAIN = RETIME ? 0 : (KIND == 2 ? 2 * R : R);
constexpr int NP1 = PF + RETAIN;                          // ring slots
constexpr int FR = (NIN * PL + NTHR - 1) / NTHR;          // ld/st prefetch fragment

__device__ __forceinline__ void kernel_stream1(const cst_kparams& P, double* smem) {
  Ctx C{P};
  constexpr int D = PF;
  constexpr int NP = STAGING == 1 ? 1 : NP1;
  const SGeo g = stream_geo(P);
  const int ta = thread_x();
  const int tb = SZ ? thread_y() : thread_z();
  const int tid = threadIdx.x;
  const int n_planes = (g.s_end - g.s_start) + 2 * R;
  const double* __restrict__ in = P.in[0];
  double* __restrict__ out = P.out[0];
  u64* bars = (u64*)(smem + NP * RSLOT);

  int la[NCA], lb[NCB];
#pragma unroll
  for (int i = 0; i < NCA; ++i) la[i] = merged_pos(i, ta, TBA, BMA);
#pragma unroll
  for (int i = 0; i < NCB; ++i) lb[i] = merged_pos(i, tb, TBB, BMB);
  const long long col0 = (long long)g.a0 + (long long)g.b0 * g.st_b;

  // retimed: acc = pending outputs (2R+1 per point); gather: queue of centre values
  double acc[NCB][NCA][W];
#pragma unroll
  for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
    for (int ia = 0; ia < NCA; ++ia)
#pragma unroll
      for (int m = 0; m < W; ++m) acc[ib][ia][m] = 0.0;

  double frag[D > 1 && STAGING == 2 ? (D - 1) * FR : 1];

  // ---- prologue: first D planes in flight
  if constexpr (STAGING == 3) {
    if (tid == 0) {
      for (int s = 0; s < NP; ++s) {
        mbar_init(&bars[s], 1);  // full: producer arrive + TMA bytes
#if CST_EMPTY_BARRIERS
        mbar_init(&bars[NP + s], NTHR / 32);  // empty: one arrive per warp
#endif
      }
      fence_mbar_init();
    }
    __syncthreads();
    if (tid == 0) {
      for (int j = 0; j < D && j < n_planes; ++j) {
        mbar_arrive_expect_tx(&bars[j % NP], TX_BYTES);
        tma_plane(P, g, smem + (j % NP) * RSLOT, &bars[j % NP], g.s_start - R + j);
      }
    }
  } else if constexpr (STAGING == 2) {
    ldst_plane(P, g, smem, g.s_start - R);
    if constexpr (D > 1) {
#pragma unroll
      for (int f = 0; f < D - 1; ++f)
#pragma unroll
        for (int q = 0; q < FR; ++q) {
          const int e = tid + q * NTHR;
          frag[f * FR + q] =
              (e < NIN * PL && 1 + f < n_planes) ? plane_elem(P, g, e, g.s_start - R + 1 + f) : 0.0;
        }
    }
    __syncthreads();
  }

  auto plane_ld = [&](int slot, int p) {
    if constexpr (STAGING == 1)
      return GlobPlane{in + col0 + (long long)p * g.st_s, g.st_b};
    else
      return SmemPlane{smem + slot * RSLOT};
  };
  auto store = [&](int ib, int ia, int po, double v) {
    if (g.a0 + la[ia] < g.n_a && g.b0 + lb[ib] < g.n_b)
    {
      const long long off = col0 + la[ia] + (long long)lb[ib] * g.st_b + (long long)po * g.st_s;
      out[off] = v;
      if constexpr (CST_REMOTE) P.rout[0][off] = v;
    }
  };

#pragma unroll(UFS)
  for (int j0 = 0; j0 < n_planes; j0 += W) {
    static_for<0, W>([&](auto UU) {
      constexpr int u = decltype(UU)::value;
      const int j = j0 + u;
      if (j >= n_planes) return;  // CTA-uniform
      const int p = g.s_start - R + j;
      const int slot = j % NP;
      if constexpr (STAGING == 3) mbar_wait(&bars[slot], (u32)((j / NP) & 1));

      if constexpr (KIND == 1 && RETIME) {
        // retiming: plane p adds ws[p-o]*u to outputs o = p-R..p+R, its in-plane
        // part to output p; output p-R is then complete.   logical m -> phys (m+u)%W
        star_retimed_plane<u>(C, plane_ld(slot, p), la, lb, acc);
        if (j >= 2 * R) {
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) store(ib, ia, p - R, acc[ib][ia][u % W]);
        }
#pragma unroll
        for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
          for (int ia = 0; ia < NCA; ++ia) acc[ib][ia][u % W] = 0.0;
      } else if constexpr (KIND == 1) {
        // gather: register queue of the 2R+1 centre values (2.5-D blocking)
        // logical q[m] (plane p-2R+m) -> phys (m+u+1)%W ; newest (m = 2R) -> phys u
        {
          double cen[NCB][NCA];
          load_centres(plane_ld(slot, p), la, lb, cen);
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) acc[ib][ia][u % W] = cen[ib][ia];
        }
        if (j >= 2 * R) {
          const int po = p - R;
          double ip[NCB][NCA], cen[NCB][NCA];
          star_inplane(C, plane_ld((j - R) % NP, po), la, lb, ip, cen);
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) {
              double s = ip[ib][ia];
#pragma unroll
              for (int k = -R; k <= R; ++k)
                if (k != 0) s = fma(C.coef(star_ci(AX_S, k)), acc[ib][ia][(R + k + u + 1) % W], s);
              store(ib, ia, po, s);
            }
        }
      } else if constexpr (KIND == 2 && RETIME) {
        // box retimed: slices ds = +1, 0, -1 of plane p go to outputs p-1, p, p+1
        double S[3][NCB][NCA];
#pragma unroll
        for (int q = 0; q < 3; ++q)
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) S[q][ib][ia] = 0.0;
        box_slices<3, R, -1>(C, plane_ld(slot, p), la, lb, S);
#pragma unroll
        for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
          for (int ia = 0; ia < NCA; ++ia)
#pragma unroll
            for (int m = 0; m < W; ++m) acc[ib][ia][(m + u) % W] += S[m][ib][ia];
        if (j >= 2 * R) {
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) store(ib, ia, p - R, acc[ib][ia][u % W]);
        }
#pragma unroll
        for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
          for (int ia = 0; ia < NCA; ++ia) acc[ib][ia][u % W] = 0.0;
      } else if constexpr (KIND == 2) {
        // box gather: one chain over planes o-1, o, o+1 (oracle order dz, dy, dx)
        if (j >= 2 * R) {
          const int po = p - R;
          double S[1][NCB][NCA];
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) S[0][ib][ia] = 0.0;
          static_for<0, W>([&](auto QQ) {
            constexpr int ds = decltype(QQ)::value - R;
            box_slices<1, ds, 0>(C, plane_ld((j - R + ds) % NP, po + ds), la, lb, S);
          });
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) store(ib, ia, po, S[0][ib][ia]);
        }
      }

      // ---- release the oldest live slot and refill it with plane j + D
      if constexpr (STAGING == 3) {
#if CST_EMPTY_BARRIERS
        // per-warp release on an "empty" mbarrier; only the producer waits (experimental)
        if (j >= RETAIN) {
          __syncwarp();
          if ((tid & 31) == 0) mbar_arrive(&bars[NP + (j - RETAIN) % NP]);
        }
        if (tid == 0 && j + D < n_planes) {
          const int jn = j + D, sl = jn % NP;
          if (jn >= NP) mbar_wait(&bars[NP + sl], (u32)((jn / NP - 1) & 1));
#else
        // CTA barrier: every warp is done with the slot of plane j - RETAIN, which is then
        // refilled with plane j + D
        __syncthreads();
        if (tid == 0 && j + D < n_planes) {
          const int sl = (j + D) % NP;
#endif
          fence_proxy_async();
          mbar_arrive_expect_tx(&bars[sl], TX_BYTES);
          tma_plane(P, g, smem + sl * RSLOT, &bars[sl], p + D);
        }
      } else if constexpr (STAGING == 2) {
        __syncthreads();
        if (j + 1 < n_planes) {
          double* dst = smem + ((j + 1) % NP) * RSLOT;
          if constexpr (D == 1) {
            ldst_plane(P, g, dst, p + 1);
          } else {
#pragma unroll
            for (int q = 0; q < FR; ++q) {
              const int e = tid + q * NTHR;
              if (e < NIN * PL) dst[(e / PL) * SLOT + e % PL] = frag[q];
            }
#pragma unroll
            for (int f = 0; f < D - 2; ++f)
#pragma unroll
              for (int q = 0; q < FR; ++q) frag[f * FR + q] = frag[(f + 1) * FR + q];
#pragma unroll
            for (int q = 0; q < FR; ++q) {
              const int e = tid + q * NTHR;
              frag[(D - 2) * FR + q] =
                  (e < NIN * PL && j + D < n_planes) ? plane_elem(P, g, e, p + D) : 0.0;
            }
          }
        }
        __syncthreads();
      }
    });
  }
}


// =============================================================================
// hypterm-like fast streaming path, T_SD == 1 (Table III "hypterm")
//   directions: a = x, b = other in-plane dim, s = streamed dim
//   in-plane terms T_a, T_b from register-blocked windows of the staged plane;
//   streamed-direction terms from per-plane products E_f scattered into 2R+1 pending
//   outputs (retiming) or gathered from a 2R+1 register queue.
// =============================================================================
constexpr int DA = 0, DB = SZ ? 1 : 2, DS = SZ ? 2 : 1;  // direction (0 x, 1 y, 2 z)

// derivative weight of offset k along direction dir (hypterm, R = 4):
//   w_d[k] = -sign(k) dxinv_d a_|k|, from the bank's products P_d[j] = dxinv_d a_j
//   (j = 1..R; host cst_api.cpp: after the 7 user coefficients, d = z, y, x); the
//   negation is exact, so every use is bit-identical to a stored signed table
__host__ __device__ constexpr int ws_base(int dir) { return 7 + R * (dir == 2 ? 0 : (dir == 1 ? 1 : 2)); }
__device__ __forceinline__ double hws(const Ctx& C, int dir, int k) {
  const double p = C.coef(ws_base(dir) + (k < 0 ? -k : k) - 1);
  return k > 0 ? -p : p;
}

// load a line of values through the point block: along a (x-window of row lb, starting
// la - XR, length BMA + 2XR) or along b (column la, rows lb - R .., length BMB + 2R)
template <int AXIS, class LD>
__device__ __forceinline__ void load_line(const LD& ld, int la, int lb, double* w) {
  if constexpr (AXIS == 0) {
    load_xwin(ld, la, lb, w);
  } else {
#pragma unroll
    for (int q = 0; q < BMB + 2 * R; ++q) {
      if (BMB == 1 && q == R) {  // the point itself: derivative terms never read it
        w[q] = 0.0;
        continue;
      }
      w[q] = ld.at(la, lb - R + q);
    }
  }
}

// T_d[f] (d = DIR, f = 0..4) for the thread's points, d in {a, b}:
//   T_d[f] = dxinv_d * sum_k a_k e_k[f]   (k = 1..4 ascending, oracle term order)
template <int AXIS, class LD>
__device__ __forceinline__ void hyp_inplane(const Ctx& C, const LD* ld, const int* la,
                                            const int* lb, double (&t)[5][NCB][NCA]) {
  constexpr int DIR = AXIS == 0 ? DA : DB;
  constexpr int QD = 4 + DIR;
  constexpr int LEN = AXIS == 0 ? BMA + 2 * XR : BMB + 2 * R;
  constexpr int OFF = AXIS == 0 ? XR : R;          // window index of the run's first point
  constexpr int NL = AXIS == 0 ? NCB * CMA : NCA * CMB;  // lines
  constexpr int NPL = AXIS == 0 ? BMA : BMB;             // points per line
  const double dxi = C.coef(4 + DIR);
#if CST_HYP_SCALAR
  // experimental: no windows, 12 scalar loads per k (fewer live registers)
#pragma unroll
  for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
    for (int ia = 0; ia < NCA; ++ia) {
      auto at = [&](int arr, int kk) {
        return AXIS == 0 ? ld[arr].at(la[ia] + kk, lb[ib]) : ld[arr].at(la[ia], lb[ib] + kk);
      };
      double sum[5];
#pragma unroll
      for (int k = 1; k <= 4; ++k) {
        const double qp = at(QD, k), qm = at(QD, -k), p4 = at(7, k), m4 = at(7, -k);
        const double a = C.coef(k - 1);
#pragma unroll
        for (int m = 0; m < 4; ++m) {
          const double cp = at(m, k), cm = at(m, -k);
          if (m == DIR) sum[0] = (k == 1) ? a * (cp - cm) : fma(a, cp - cm, sum[0]);
          double e = fma(cp, qp, -(cm * qm));
          if (m == 3) e = e + fma(p4, qp, -(m4 * qm));
          else if (m == DIR) e = e + (p4 - m4);
          sum[m + 1] = (k == 1) ? a * e : fma(a, e, sum[m + 1]);
        }
      }
#pragma unroll
      for (int f = 0; f < 5; ++f) t[f][ib][ia] = dxi * sum[f];
    }
  return;
#endif
#pragma unroll
  for (int line = 0; line < NL; ++line) {
    // line -> (run start la0, lb0) and point (ib, ia) of its t-th point
    const int ib0 = AXIS == 0 ? line / CMA : (line % CMB) * BMB;
    const int ia0 = AXIS == 0 ? (line % CMA) * BMA : line / CMB;
    const int la0 = la[ia0], lb0 = lb[ib0];
    double wq[LEN], w4[LEN], wc[LEN];
    load_line<AXIS>(ld[QD], la0, lb0, wq);
    load_line<AXIS>(ld[7], la0, lb0, w4);
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      // keep ptxas from hoisting all six windows at once (register budget of the
      // 45-accumulator fast path; shared-memory latency is hidden by the other warps)
      if constexpr (MINB > 1) asm volatile("" ::: "memory");
      load_line<AXIS>(ld[m], la0, lb0, wc);
#pragma unroll
      for (int pt = 0; pt < NPL; ++pt) {
        const int ib = AXIS == 0 ? ib0 : ib0 + pt;
        const int ia = AXIS == 0 ? ia0 + pt : ia0;
        const int c = OFF + pt;
        if (m == DIR) {  // mass flux: cons_d(+k) - cons_d(-k)
          double sum = 0.0;
#pragma unroll
          for (int k = 1; k <= 4; ++k) {
            const double e = wc[c + k] - wc[c - k];
            sum = (k == 1) ? C.coef(0) * e : fma(C.coef(k - 1), e, sum);
          }
          t[0][ib][ia] = dxi * sum;
        }
        double sum = 0.0;
#pragma unroll
        for (int k = 1; k <= 4; ++k) {
          double e = fma(wc[c + k], wq[c + k], -(wc[c - k] * wq[c - k]));
          if (m == 3)
            e = e + fma(w4[c + k], wq[c + k], -(w4[c - k] * wq[c - k]));
          else if (m == DIR)
            e = e + (w4[c + k] - w4[c - k]);
          sum = (k == 1) ? C.coef(0) * e : fma(C.coef(k - 1), e, sum);
        }
        t[m + 1][ib][ia] = dxi * sum;
      }
    }
  }
}

// per-plane streamed-direction products E_f at the thread's points
template <class LD>
__device__ __forceinline__ void hyp_products(const LD* ld, const int* la, const int* lb,
                                             double (&E)[5][NCB][NCA]) {
  constexpr int QS = 4 + DS;
#pragma unroll
  for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
    for (int ia = 0; ia < NCA; ++ia) {
      const double qs = ld[QS].at(la[ia], lb[ib]);
      const double q4 = ld[7].at(la[ia], lb[ib]);
      double cm[4];
#pragma unroll
      for (int m = 0; m < 4; ++m) cm[m] = ld[m].at(la[ia], lb[ib]);
      E[0][ib][ia] = cm[DS];
#pragma unroll
      for (int m = 0; m < 3; ++m) E[m + 1][ib][ia] = m == DS ? fma(cm[m], qs, q4) : cm[m] * qs;
      E[4][ib][ia] = fma(cm[3], qs, q4 * qs);
    }
}

__device__ __forceinline__ void kernel_hyp_stream1(const cst_kparams& P, double* smem) {
  Ctx C{P};
  constexpr int D = PF;
  constexpr int NP = STAGING == 1 ? 1 : NP1;
  const SGeo g = stream_geo(P);
  const int ta = thread_x();
  const int tb = SZ ? thread_y() : thread_z();
  const int tid = threadIdx.x;
  const int n_planes = (g.s_end - g.s_start) + 2 * R;
  u64* bars = (u64*)(smem + NP * RSLOT);

  int la[NCA], lb[NCB];
#pragma unroll
  for (int i = 0; i < NCA; ++i) la[i] = merged_pos(i, ta, TBA, BMA);
#pragma unroll
  for (int i = 0; i < NCB; ++i) lb[i] = merged_pos(i, tb, TBB, BMB);
  const long long col0 = (long long)g.a0 + (long long)g.b0 * g.st_b;

  // streamed-direction weights ws[k] = -sign(k) dxinv_s a_|k| (host-precomputed, in the
  // constant bank after the 7 user coefficients: 8 for s = z, then 8 for s = y):
  // plane p contributes ws[p-o] * E_f(p) to flux_f(o)
  auto ws = [&](int k) { return hws(C, DS, k); };

  double acc[5][NCB][NCA][W];  // retimed: pending fluxes ; gather: queue of E_f
#pragma unroll
  for (int f = 0; f < 5; ++f)
#pragma unroll
    for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
      for (int ia = 0; ia < NCA; ++ia)
#pragma unroll
        for (int m = 0; m < W; ++m) acc[f][ib][ia][m] = 0.0;

  double frag[D > 1 && STAGING == 2 ? (D - 1) * FR : 1];
  if constexpr (STAGING == 3) {
    if (tid == 0) {
      for (int s = 0; s < NP; ++s) {
        mbar_init(&bars[s], 1);  // full: producer arrive + TMA bytes
#if CST_EMPTY_BARRIERS
        mbar_init(&bars[NP + s], NTHR / 32);  // empty: one arrive per warp
#endif
      }
      fence_mbar_init();
    }
    __syncthreads();
    if (tid == 0) {
      for (int j = 0; j < D && j < n_planes; ++j) {
        mbar_arrive_expect_tx(&bars[j % NP], TX_BYTES);
        tma_plane(P, g, smem + (j % NP) * RSLOT, &bars[j % NP], g.s_start - R + j);
      }
    }
  } else if constexpr (STAGING == 2) {
    ldst_plane(P, g, smem, g.s_start - R);
    if constexpr (D > 1) {
#pragma unroll
      for (int f = 0; f < D - 1; ++f)
#pragma unroll
        for (int q = 0; q < FR; ++q) {
          const int e = tid + q * NTHR;
          frag[f * FR + q] =
              (e < NIN * PL && 1 + f < n_planes) ? plane_elem(P, g, e, g.s_start - R + 1 + f) : 0.0;
        }
    }
    __syncthreads();
  }

  auto loaders = [&](int slot, int p, auto* out8) {
#pragma unroll
    for (int a = 0; a < NIN; ++a) {
      if constexpr (STAGING == 1)
        out8[a] = GlobPlane{P.in[a] + col0 + (long long)p * g.st_s, g.st_b};
      else
        out8[a] = splane(smem + slot * RSLOT, a);
    }
  };
  using LDT = typename Cond<STAGING == 1, GlobPlane, SPlane>::type;
  auto store5 = [&](int ib, int ia, int po, double (&v)[5]) {
    if (g.a0 + la[ia] < g.n_a && g.b0 + lb[ib] < g.n_b) {
      const long long off = col0 + la[ia] + (long long)lb[ib] * g.st_b + (long long)po * g.st_s;
#pragma unroll
      for (int f = 0; f < 5; ++f) put(P, f, off, v[f]);
    }
  };

#pragma unroll(UFS)
  for (int j0 = 0; j0 < n_planes; j0 += W) {
    static_for<0, W>([&](auto UU) {
      constexpr int u = decltype(UU)::value;
      const int j = j0 + u;
      if (j >= n_planes) return;
      const int p = g.s_start - R + j;
      const int slot = j % NP;
      if constexpr (STAGING == 3) mbar_wait(&bars[slot], (u32)((j / NP) & 1));
      LDT ld[NIN];
      loaders(slot, p, ld);
      if constexpr (RETIME) {
        // scatter in an order that keeps few temporaries live: E_f first, then T_a, T_b
        {
          double E[5][NCB][NCA];
          hyp_products(ld, la, lb, E);
#pragma unroll
          for (int f = 0; f < 5; ++f)
#pragma unroll
            for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
              for (int ia = 0; ia < NCA; ++ia)
#pragma unroll
                for (int m = 0; m < W; ++m) {
                  if (m == R) continue;
                  double& a = acc[f][ib][ia][(m + u) % W];
                  a = fma(ws(R - m), E[f][ib][ia], a);  // k = p - o = R - m
                }
        }
        {
          double t[5][NCB][NCA];
          hyp_inplane<0>(C, ld, la, lb, t);
#pragma unroll
          for (int f = 0; f < 5; ++f)
#pragma unroll
            for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
              for (int ia = 0; ia < NCA; ++ia) acc[f][ib][ia][(R + u) % W] -= t[f][ib][ia];
        }
        {
          double t[5][NCB][NCA];
          hyp_inplane<1>(C, ld, la, lb, t);
#pragma unroll
          for (int f = 0; f < 5; ++f)
#pragma unroll
            for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
              for (int ia = 0; ia < NCA; ++ia) acc[f][ib][ia][(R + u) % W] -= t[f][ib][ia];
        }
        if (j >= 2 * R) {
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) {
              double v[5];
#pragma unroll
              for (int f = 0; f < 5; ++f) v[f] = acc[f][ib][ia][u % W];
              store5(ib, ia, p - R, v);
            }
        }
#pragma unroll
        for (int f = 0; f < 5; ++f)
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) acc[f][ib][ia][u % W] = 0.0;
      } else {
        // gather: queue of E_f, newest at phys u
        double E[5][NCB][NCA];
        hyp_products(ld, la, lb, E);
#pragma unroll
        for (int f = 0; f < 5; ++f)
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) acc[f][ib][ia][u % W] = E[f][ib][ia];
        if (j >= 2 * R) {
          const int po = p - R;
          LDT ldo[NIN];
          loaders((j - R) % NP, po, ldo);
          double ta_[5][NCB][NCA], tb_[5][NCB][NCA];
          hyp_inplane<0>(C, ldo, la, lb, ta_);
          hyp_inplane<1>(C, ldo, la, lb, tb_);
          const double dxs = C.coef(4 + DS);
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int ia = 0; ia < NCA; ++ia) {
              double v[5];
#pragma unroll
              for (int f = 0; f < 5; ++f) {
                double sum = 0.0;
#pragma unroll
                for (int k = 1; k <= R; ++k) {
                  const double e = acc[f][ib][ia][(R + k + u + 1) % W] -
                                   acc[f][ib][ia][(R - k + u + 1) % W];
                  sum = (k == 1) ? C.coef(0) * e : fma(C.coef(k - 1), e, sum);
                }
                v[f] = -ta_[f][ib][ia] - tb_[f][ib][ia] - dxs * sum;
              }
              store5(ib, ia, po, v);
            }
        }
      }

      if constexpr (STAGING == 3) {
#if CST_EMPTY_BARRIERS
        // per-warp release on an "empty" mbarrier; only the producer waits (experimental)
        if (j >= RETAIN) {
          __syncwarp();
          if ((tid & 31) == 0) mbar_arrive(&bars[NP + (j - RETAIN) % NP]);
        }
        if (tid == 0 && j + D < n_planes) {
          const int jn = j + D, sl = jn % NP;
          if (jn >= NP) mbar_wait(&bars[NP + sl], (u32)((jn / NP - 1) & 1));
#else
        // CTA barrier: every warp is done with the slot of plane j - RETAIN, which is then
        // refilled with plane j + D
        __syncthreads();
        if (tid == 0 && j + D < n_planes) {
          const int sl = (j + D) % NP;
#endif
          fence_proxy_async();
          mbar_arrive_expect_tx(&bars[sl], TX_BYTES);
          tma_plane(P, g, smem + sl * RSLOT, &bars[sl], p + D);
        }
      } else if constexpr (STAGING == 2) {
        __syncthreads();
        if (j + 1 < n_planes) {
          double* dst = smem + ((j + 1) % NP) * RSLOT;
          if constexpr (D == 1) {
            ldst_plane(P, g, dst, p + 1);
          } else {
#pragma unroll
            for (int q = 0; q < FR; ++q) {
              const int e = tid + q * NTHR;
              if (e < NIN * PL) dst[(e / PL) * SLOT + e % PL] = frag[q];
            }
#pragma unroll
            for (int f = 0; f < D - 2; ++f)
#pragma unroll
              for (int q = 0; q < FR; ++q) frag[f * FR + q] = frag[(f + 1) * FR + q];
#pragma unroll
            for (int q = 0; q < FR; ++q) {
              const int e = tid + q * NTHR;
              frag[(D - 2) * FR + q] =
                  (e < NIN * PL && j + D < n_planes) ? plane_elem(P, g, e, p + D) : 0.0;
            }
          }
        }
        __syncthreads();
      }
    });
  }
}

// =============================================================================
// generic streaming path (any kind, any T_SD): ring of D*TS + 2R planes, gather
// =============================================================================
__device__ __forceinline__ void kernel_stream_generic(const cst_kparams& P, double* smem) {
  Ctx C{P};
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
  u64* bars = (u64*)(smem + NP * RSLOT);

  auto issue = [&](int j) {  // load plane j (sequence index) into its slot
    if (j >= n_planes) return;
    const int sl = j % NP;
    if constexpr (STAGING == 3) {
      if (tid == 0) {
        fence_proxy_async();
        mbar_arrive_expect_tx(&bars[sl], TX_BYTES);
        tma_plane(P, g, smem + sl * RSLOT, &bars[sl], g.s_start - R + j);
      }
    } else if constexpr (STAGING == 2) {
      ldst_plane(P, g, smem + sl * RSLOT, g.s_start - R + j);
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
        const int lbp = merged_pos(ib, tb, TBB, BMB);
        if constexpr (PAIRED) {
          // rhs4, BM_x = 2: the thread's two x-adjacent points in lockstep; every smem
          // operand is one 16-B load for both (odd x-offsets combine the two aligned
          // neighbours, which the even offsets load anyway)
          const int lap = merged_pos(0, ta, TBA, BMA);
          const int a = g.a0 + lap, b = g.b0 + lbp;
          if (a >= g.n_a || b >= g.n_b || s >= g.s_end) continue;
          const long long off = a + b * g.st_b + (long long)s * g.st_s;
          const int jp = s - g.s_start + R;
          auto U2 = [&](int arr, int dx, int dy, int dz) {
            const int db = SZ ? dy : dz, ds = SZ ? dz : dy;
            const double* row = smem + ((jp + ds) % NP) * RSLOT + arr * SLOT +
                                (lbp + R + db) * PA + lap + XR;
            if ((dx & 1) == 0) {
              const double2 v = *reinterpret_cast<const double2*>(row + dx);
              return dpair{v.x, v.y};
            }
            const double2 lo = *reinterpret_cast<const double2*>(row + dx - 1);
            const double2 hi = *reinterpret_cast<const double2*>(row + dx + 1);
            return dpair{lo.y, hi.x};
          };
          dpair o2[3];
          rhs4_point_t<dpair>(C, U2, o2);
#pragma unroll
          for (int q = 0; q < NOUT; ++q) {
            put(P, q, off, o2[q].x);
            if (a + 1 < g.n_a) put(P, q, off + 1, o2[q].y);
          }
          continue;
        }
#pragma unroll(UFA)
        for (int ia = 0; ia < BMA * CMA; ++ia) {
          const int lap = merged_pos(ia, ta, TBA, BMA);
          const int a = g.a0 + lap, b = g.b0 + lbp;
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
              return smem[((jp + ds) % NP) * RSLOT + arr * SLOT + (lbp + R + db) * PA +
                          lap + XR + da];
            };
            point(C, U, o);
          }
#pragma unroll
          for (int q = 0; q < NOUT; ++q) put(P, q, off, o[q]);
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
// rhs4center-like, retimed column walk (NEXT-1; use_retiming = 2 with T_SD = 1, TMA,
// CM = 1, BM_b = 1, BM_a <= 2).  Retiming applied to the operator of
// reading O7: every mixed term D_o[c D_n f] is split by where its two derivatives point.
//   outer along s (D_s[mu D_a u_s], D_s[mu D_b u_s], D_s[la D_a u_a], D_s[la D_b u_b]):
//     the inner product P = c D_n f is formed once per plane at the point's own column (its
//     operands are the in-plane windows the V terms load anyway) and scattered into the
//     pending outputs c-2, c-1, c+1, c+2 with the outer weights (-1, 8, -8, 1);
//   inner along s (D_a[la D_s u_s], D_b[la D_s u_s], D_a[mu D_s u_a], D_b[mu D_s u_b]):
//     the products Q = c D_s f of plane c are formed once per column from the s-window and
//     staged as three product planes in shared memory (own columns by their threads, the
//     cross-shaped halo columns from the ring), then differenced along a / b;
//   both derivatives in-plane: gathered from the ring plane as in the generic path.
// The s-window of the own column (u1..u3, mu, lambda at planes c-2..c+2): a register queue
// of u1..u3 with mu / lambda from the ring (one point per thread; 2.5-D blocking), read
// from the ring (two x-adjacent points per thread), or a tensor-memory queue (qstore = 2).
// At step c the newest plane is c+2; output c-2 completes.
// =============================================================================
constexpr bool R4RET = KIND == 4 && STREAM && TS == 1 && RETIME;
constexpr int R4NP = PF + 2 * R;                 // ring: planes c-2 .. c+2 + PF-1 ahead
constexpr int R4NH = 2 * TB + 4 * (TA / 2);      // halo column pairs of the product planes
// the two x-adjacent points of a BM_a = 2 thread in lockstep (every smem operand one 16-B
// load for both); their s-windows come from the ring (a register queue spills them: 255
// registers + 200 B of stack); one point per thread keeps u1..u3 in registers (166 registers,
// 3 CTAs/SM; all five: 216 registers, 2 CTAs, 15 % slower).  Experiment hook: CST_R4Q.
#ifndef CST_R4Q
#define CST_R4Q (BMA == 1 ? 3 : 0)
#endif
constexpr int R4Q = QTM ? 0 : CST_R4Q;  // arrays of the s-window in the register queue
// qstore = 2: the whole s-window queue (5 arrays x 5 planes) lives in tensor memory, one lane
// per thread (R15): R4TC columns per value, R4TPT per thread (array-major, 5 slots each)
constexpr int R4TC = BMA == 2 ? 4 : 2, R4TPT = 25 * R4TC;
constexpr int R4TUSED = ((NTHR / 32 + 3) / 4) * R4TPT;
constexpr int R4TCOLS = R4TUSED <= 32 ? 32 : R4TUSED <= 64 ? 64 : R4TUSED <= 128 ? 128
                       : R4TUSED <= 256 ? 256 : 512;
// one value T of the queue (array-major layout: column of array a, slot p =
// tq + (a * 5 + p) * R4TC): store / load into raw 32-bit words / unpack
template <class T>
__device__ __forceinline__ void r4_tm_st1(u32 a, T v) {
  if constexpr (sizeof(T) == 8) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};" ::"r"(a),
                 "r"((u32)__double2loint(v)), "r"((u32)__double2hiint(v)));
  } else {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a),
                 "r"((u32)__double2loint(v.x)), "r"((u32)__double2hiint(v.x)),
                 "r"((u32)__double2loint(v.y)), "r"((u32)__double2hiint(v.y)));
  }
}
__device__ __forceinline__ void tmem_ld_x4(u32 a, u32* r) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(a)
               : "memory");
}
template <class T>
__device__ __forceinline__ void r4_tm_ld1(u32 a, u32* r) {
  if constexpr (sizeof(T) == 8) tmem_ld_x2(a, r);
  else tmem_ld_x4(a, r);
}
template <class T>
__device__ __forceinline__ T r4_tm_v1(const u32* r) {
  if constexpr (sizeof(T) == 8) return tmem_d(r[0], r[1]);
  else return T{tmem_d(r[0], r[1]), tmem_d(r[2], r[3])};
}

template <class T>
__device__ __forceinline__ T r4_row(const double* row, int da) {
  if constexpr (sizeof(T) == 8) {
    return row[da];
  } else {
    if ((da & 1) == 0) {
      const double2 v = *reinterpret_cast<const double2*>(row + da);
      return T{v.x, v.y};
    }
    const double2 lo = *reinterpret_cast<const double2*>(row + da - 1);
    const double2 hi = *reinterpret_cast<const double2*>(row + da + 1);
    return T{lo.y, hi.x};
  }
}
template <class T>
__device__ __forceinline__ void r4_put_row(double* row, T v) {
  if constexpr (sizeof(T) == 8) row[0] = v;
  else *reinterpret_cast<double2*>(row) = make_double2(v.x, v.y);
}
__device__ __forceinline__ double r4_lane(double v, int) { return v; }
__device__ __forceinline__ double r4_lane(dpair v, int h) { return h ? v.y : v.x; }

// V_d[a](f) of reading O7, unscaled (the 1/6 and s_d^2 are in coefficient 3 + d)
template <class T, class A, class F>
__device__ __forceinline__ T r4_v(const A& a, const F& f) {
  const T am2 = a(-2), am1 = a(-1), a0 = a(0), ap1 = a(1), ap2 = a(2);
  const T m1 = fma(-0.75, a0 + am2, am1);
  const T m2 = fma(3.0, a0 + am1, am2 + ap1);
  const T m3 = fma(3.0, ap1 + a0, am1 + ap2);
  const T m4 = fma(-0.75, a0 + ap2, ap1);
  const T f0 = f(0);
  T v = m1 * (f(-2) - f0);
  v = fma(m2, f(-1) - f0, v);
  v = fma(m3, f(1) - f0, v);
  v = fma(m4, f(2) - f0, v);
  return v;
}
// the same split in two: the weights m1..m4 of a field a, then the sum over f
template <class T, class A>
__device__ __forceinline__ void r4_m(const A& a, T (&m)[4]) {
  const T am2 = a(-2), am1 = a(-1), a0 = a(0), ap1 = a(1), ap2 = a(2);
  m[0] = fma(-0.75, a0 + am2, am1);
  m[1] = fma(3.0, a0 + am1, am2 + ap1);
  m[2] = fma(3.0, ap1 + a0, am1 + ap2);
  m[3] = fma(-0.75, a0 + ap2, ap1);
}
template <class T, class F>
__device__ __forceinline__ T r4_vm(const T (&m)[4], const F& f) {
  const T f0 = f(0);
  T v = m[0] * (f(-2) - f0);
  v = fma(m[1], f(-1) - f0, v);
  v = fma(m[2], f(1) - f0, v);
  v = fma(m[3], f(2) - f0, v);
  return v;
}
// unscaled D'[f] = 8 (f(+1) - f(-1)) + (f(-2) - f(+2))  (the 1/12 factors are folded)
template <class T, class F>
__device__ __forceinline__ T r4_d(const F& f) {
  return fma(8.0, f(1) - f(-1), f(-2) - f(2));
}

template <int DUMMY>
__device__ __forceinline__ void kernel_rhs4_ret(const cst_kparams& P, double* smem) {
  using T = typename Cond<BMA == 2, dpair, double>::type;
  static_assert(STAGING == 3 && BMA <= 2 && NCB == 1 && CMA == 1, "R16: rhs4 retimed path");
  Ctx C{P};
  constexpr int NP = R4NP;
  constexpr int QN = 5;  // s-window / pending outputs: planes c-2 .. c+2
  const SGeo g = stream_geo(P);
  const int tid = threadIdx.x;
  const int la = thread_x() * BMA;
  const int lb = SZ ? thread_y() : thread_z();
  const int n_out = g.s_end - g.s_start;
  const int n_planes = n_out + 2 * R;
  double* qbuf = smem + NP * RSLOT;  // 2 buffers x {la*D_s u_s, mu*D_s u_a, mu*D_s u_b}
  u64* bars = (u64*)(qbuf + 6 * SLOT);
  const int own = (lb + R) * PA + la + XR;  // the point's element in a plane slot
  auto slot = [&](int j) { return smem + (j % NP) * RSLOT; };
  const double kv[3] = {C.coef(3), C.coef(4), C.coef(5)};
  auto wp = [&](int d, int i) { return C.coef(6 + d + i - 1); };  // s_d s_i / 144, d != i

  u32* tslot = (u32*)(bars + NP);  // spare mbarrier words (kernel_smem_bytes reserves 2 NP)
  const int warp = tid >> 5;
  if constexpr (QTM) {
    if (warp == 0) tmem_alloc(tslot, R4TCOLS);
  }
  if (tid == 0) {
    for (int s = 0; s < NP; ++s) mbar_init(&bars[s], 1);
    fence_mbar_init();
  }
  if constexpr (QTM) tmem_fence_before_sync();
  __syncthreads();
  if constexpr (QTM) tmem_fence_after_sync();
  // the thread's TMEM queue: lane quarter of its warp, column block of its warp in the quarter
  const u32 tq = QTM ? *tslot + ((u32)((warp & 3) * 32) << 16) + (u32)((warp >> 2) * R4TPT) : 0u;
  if (tid == 0) {
    for (int j = 0; j < NP && j < n_planes; ++j) {
      mbar_arrive_expect_tx(&bars[j], TX_BYTES);
      tma_plane(P, g, slot(j), &bars[j], g.s_start - R + j);
    }
  }

  // queue q[arr][phys]: logical k (plane c-2+k) at phys (k + u) % 5 in phase u = c % 5
  constexpr int NQA = R4Q;
  T q[NQA > 0 ? NQA : 1][QN];
  T acc[3][QN];  // pending outputs, same rotation; index = physical output direction
#pragma unroll
  for (int m = 0; m < QN; ++m) {
#pragma unroll
    for (int i = 0; i < 3; ++i) acc[i][m] = T{};
#pragma unroll
    for (int a = 0; a < NQA; ++a) q[a][m] = T{};
  }
  // prologue: planes 0 and 1 are logical 2 and 3 of step 0
  for (int j = 0; j < 2 && j < n_planes; ++j) {
    mbar_wait(&bars[j], 0u);
#pragma unroll
    for (int a = 0; a < NQA; ++a) q[a][2 + j] = r4_row<T>(slot(j) + a * SLOT + own, 0);
    if constexpr (QTM) {
#pragma unroll
      for (int a = 0; a < 5; ++a)
        r4_tm_st1<T>(tq + (u32)((a * QN + 2 + j) * R4TC), r4_row<T>(slot(j) + a * SLOT + own, 0));
    }
  }
  if constexpr (QTM) tmem_wait_st();

  const long long col = (long long)(g.a0 + la) + (long long)(g.b0 + lb) * g.st_b;
  const bool in_b = g.b0 + lb < g.n_b;
  const bool in_a0 = g.a0 + la < g.n_a, in_a1 = BMA == 2 && g.a0 + la + 1 < g.n_a;

  for (int j0 = 0; j0 < n_planes; j0 += QN) {
    static_for<0, QN>([&](auto UU) {
      constexpr int u = decltype(UU)::value;
      auto ph = [](int k) { return (k + u) % QN; };
      const int c = j0 + u;  // centre plane (sequence index)
      if (c >= n_planes) return;  // CTA-uniform
      const bool real = c >= R && c < R + n_out;
      // ---- newest plane c+2 -> queue
      T nw[QTM ? 5 : 1];
      if (c + 2 < n_planes) {
        mbar_wait(&bars[(c + 2) % NP], (u32)(((c + 2) / NP) & 1));
#pragma unroll
        for (int a = 0; a < NQA; ++a) q[a][ph(4)] = r4_row<T>(slot(c + 2) + a * SLOT + own, 0);
        if constexpr (QTM) {
#pragma unroll
          for (int a = 0; a < 5; ++a) {
            nw[a] = r4_row<T>(slot(c + 2) + a * SLOT + own, 0);
            r4_tm_st1<T>(tq + (u32)((a * QN + ph(4)) * R4TC), nw[a]);
          }
        }
      }
      // s-window of array a at the own column, offset k in -2..2
      auto sw = [&](int a, int k) -> T {
        if (a < NQA) return q[a][ph(2 + k)];
        return r4_row<T>(slot(c + k) + a * SLOT + own, 0);
      };
      double* qb = qbuf + (c & 1) * 3 * SLOT;
      if (QTM && real) {
        // ---- V_s and the inner-s products from the TMEM queue, in stages (mu, lambda and
        // u_s; then u_a; then u_b — each load issued one stage ahead) so that only one
        // array's window is live beside the V weights
        auto tcol = [&](int a, int k) { return tq + (u32)((a * QN + ph(2 + k)) * R4TC); };
        u32 wm[4][R4TC], wl[4][R4TC], wu[3][4][R4TC];
        auto issue_u = [&](int ii, int a) {
#pragma unroll
          for (int k = 0; k < 4; ++k) r4_tm_ld1<T>(tcol(a, k - 2), wu[ii][k]);
        };
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          r4_tm_ld1<T>(tcol(3, k - 2), wm[k]);
          r4_tm_ld1<T>(tcol(4, k - 2), wl[k]);
        }
        issue_u(0, DS);
        tmem_wait_ld();
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          tmem_pin(wm[k]);
          tmem_pin(wl[k]);
          tmem_pin(wu[0][k]);
        }
        auto mu = [&](int k) { return k == 2 ? nw[3] : r4_tm_v1<T>(wm[k + 2]); };
        auto lam = [&](int k) { return k == 2 ? nw[4] : r4_tm_v1<T>(wl[k + 2]); };
        const T mu0 = mu(0), la0 = lam(0);
        // V weights for a = mu (outputs i != s) and a = 2 mu + lambda (output s)
        T mm[4], mk[4];
        r4_m<T>([&](int k) { return mu(k); }, mm);
        r4_m<T>([&](int k) { return fma(2.0, mu(k), lam(k)); }, mk);
#pragma unroll
        for (int ii = 0; ii < 3; ++ii) {
          const int i = ii == 0 ? DS : (ii == 1 ? DA : DB);
          if (ii < 2) issue_u(ii + 1, ii == 0 ? DA : DB);
          auto f = [&](int k) { return k == 2 ? nw[i] : r4_tm_v1<T>(wu[ii][k + 2]); };
          acc[i][ph(2)] = fma(kv[DS], r4_vm<T>(ii == 0 ? mk : mm, f), acc[i][ph(2)]);
          r4_put_row<T>(qb + ii * SLOT + own, (ii == 0 ? la0 : mu0) * r4_d<T>(f));
          if (ii < 2) {
            tmem_wait_ld();
#pragma unroll
            for (int k = 0; k < 4; ++k) tmem_pin(wu[ii + 1][k]);
          }
        }
      }
      if (!QTM && real) {
        // ---- V_s and the inner-s products of the own column
        const T mu0 = sw(3, 0), la0 = sw(4, 0);
#pragma unroll
        for (int i = 0; i < 3; ++i) {
          const T v = r4_v<T>(
              [&](int k) { return i == DS ? fma(2.0, sw(3, k), sw(4, k)) : sw(3, k); },
              [&](int k) { return sw(i, k); });
          acc[i][ph(2)] = fma(kv[DS], v, acc[i][ph(2)]);
        }
        r4_put_row<T>(qb + 0 * SLOT + own, la0 * r4_d<T>([&](int k) { return sw(DS, k); }));
        r4_put_row<T>(qb + 1 * SLOT + own, mu0 * r4_d<T>([&](int k) { return sw(DA, k); }));
        r4_put_row<T>(qb + 2 * SLOT + own, mu0 * r4_d<T>([&](int k) { return sw(DB, k); }));
      }
      if (real) {
        // ---- halo columns of the product planes (pairs of x-adjacent columns):
        // a-strips (la*D_s u_s, mu*D_s u_a), b-strips (la*D_s u_s, mu*D_s u_b)
        // one product per thread (la*D_s u_s by the first R4NH threads, mu*D_s u_a|b by the
        // next): the halo work is spread over twice the threads, its critical path halved
        // (0.958 vs 0.959 ms tuned, 0.980 vs 0.992 for 256 threads; profiles/r02/g31)
        for (int e2 = tid; e2 < 2 * R4NH; e2 += NTHR) {
          const int e = e2 % R4NH;
          const bool mu_part = e2 >= R4NH;  // else the lambda product
          int ha, hb, fa;
          if (e < 2 * TB) {
            ha = (e & 1) ? TA : -2;
            hb = e >> 1;
            fa = DA;
          } else {
            const int f = e - 2 * TB;
            ha = 2 * (f % (TA / 2));
            const int rr = f / (TA / 2);  // 0..3 -> rows -2, -1, TB, TB+1
            hb = rr < 2 ? rr - 2 : TB + rr - 2;
            fa = DB;
          }
          const int ho = (hb + R) * PA + ha + XR;
          auto hw = [&](int a, int k) { return r4_row<dpair>(slot(c + k) + a * SLOT + ho, 0); };
          if (!mu_part)
            r4_put_row<dpair>(qb + ho, hw(4, 0) * r4_d<dpair>([&](int k) { return hw(DS, k); }));
          else
            r4_put_row<dpair>(qb + (fa == DA ? 1 : 2) * SLOT + ho,
                              hw(3, 0) * r4_d<dpair>([&](int k) { return hw(fa, k); }));
        }
      }
      __syncthreads();
      // ---- the slot of plane c-2 is free: refill it with plane c-2+NP
      if (tid == 0 && c >= 2 && c - 2 + NP < n_planes) {
        const int jn = c - 2 + NP;
        fence_proxy_async();
        mbar_arrive_expect_tx(&bars[jn % NP], TX_BYTES);
        tma_plane(P, g, slot(jn), &bars[jn % NP], g.s_start - R + jn);
      }
      // ---- plane c, in-plane operands
      const double* pl = slot(c) + own;
      auto L = [&](int a, int da, int db) { return r4_row<T>(pl + a * SLOT + db * PA, da); };
      auto Ld = [&](int a, int dir, int k) {  // along physical direction a (x) or b
        return dir == DA ? L(a, k, 0) : L(a, 0, k);
      };
      // per in-plane direction d: the outer-s products P = c * D'_d f, scattered to outputs
      // c-2, c-1, c+1, c+2, and V_d of every output (real outputs only).  (Compiler fences
      // between these phases cut the pair variant from 228 to 168 registers but cost 10-30 %:
      // the hoisted loads are the latency hiding.)
      auto scat = [&](int i, double w, T p) {
        acc[i][ph(0)] = fma(-w, p, acc[i][ph(0)]);
        acc[i][ph(1)] = fma(8.0 * w, p, acc[i][ph(1)]);
        acc[i][ph(3)] = fma(-8.0 * w, p, acc[i][ph(3)]);
        acc[i][ph(4)] = fma(w, p, acc[i][ph(4)]);
      };
#pragma unroll
      for (int dd = 0; dd < 2; ++dd) {
        const int d = dd == 0 ? DA : DB;
        const T mu0 = L(3, 0, 0), la0 = L(4, 0, 0);
        // mu D_d u_s -> r_d ; la D_d u_d -> r_s
        scat(d, wp(d, DS), mu0 * r4_d<T>([&](int k) { return Ld(DS, d, k); }));
        scat(DS, wp(d, DS), la0 * r4_d<T>([&](int k) { return Ld(d, d, k); }));
        if (real) {
#pragma unroll
          for (int i = 0; i < 3; ++i) {
            const T v = r4_v<T>(
                [&](int k) { return i == d ? fma(2.0, Ld(3, d, k), Ld(4, d, k)) : Ld(3, d, k); },
                [&](int k) { return Ld(i, d, k); });
            acc[i][ph(2)] = fma(kv[d], v, acc[i][ph(2)]);
          }
        }
      }
      if (real) {
        // in-plane mixed terms: D_o[c D_n f] with o, n in {a, b}
        auto mixed = [&](int o, int n, int ca, int fa) {
          auto inner = [&](int ko) {
            auto f = [&](int kn) {
              return L(fa, (o == DA ? ko : 0) + (n == DA ? kn : 0),
                       (o == DB ? ko : 0) + (n == DB ? kn : 0));
            };
            return L(ca, o == DA ? ko : 0, o == DB ? ko : 0) * r4_d<T>(f);
          };
          return r4_d<T>(inner);
        };
        const double wab = wp(DA, DB);
        acc[DA][ph(2)] = fma(wab, mixed(DB, DA, 3, DB) + mixed(DA, DB, 4, DB), acc[DA][ph(2)]);
        acc[DB][ph(2)] = fma(wab, mixed(DA, DB, 3, DA) + mixed(DB, DA, 4, DA), acc[DB][ph(2)]);
        // inner-s terms: outer differences of the product planes
        const double* qp = qb + own;
        auto Q = [&](int qi, int dir, int k) {
          const double* row = qp + qi * SLOT + (dir == DB ? k * PA : 0);
          return r4_row<T>(row, dir == DA ? k : 0);
        };
        const double was = wp(DA, DS), wbs = wp(DB, DS);
        acc[DA][ph(2)] = fma(was, r4_d<T>([&](int k) { return Q(0, DA, k); }), acc[DA][ph(2)]);
        acc[DB][ph(2)] = fma(wbs, r4_d<T>([&](int k) { return Q(0, DB, k); }), acc[DB][ph(2)]);
        acc[DS][ph(2)] = fma(was, r4_d<T>([&](int k) { return Q(1, DA, k); }), acc[DS][ph(2)]);
        acc[DS][ph(2)] = fma(wbs, r4_d<T>([&](int k) { return Q(2, DB, k); }), acc[DS][ph(2)]);
      }
      // ---- output c-2 is complete
      const int co = c - 2;
      if (co >= R && co < R + n_out && in_b) {
        const long long off = col + (long long)(g.s_start + co - R) * g.st_s;
#pragma unroll
        for (int i = 0; i < 3; ++i) {
          if (in_a0) put(P, i, off, r4_lane(acc[i][ph(0)], 0));
          if (in_a1) put(P, i, off + 1, r4_lane(acc[i][ph(0)], 1));
        }
      }
#pragma unroll
      for (int i = 0; i < 3; ++i) acc[i][ph(0)] = T{};
      if constexpr (QTM) tmem_wait_st();  // the next plane reads the slot written here
    });
  }
  if constexpr (QTM) {
    tmem_fence_before_sync();
    __syncthreads();
    tmem_fence_after_sync();
    if (warp == 0) tmem_dealloc(*tslot, R4TCOLS);
  }
}

// =============================================================================
// temporal blocking, bt > 1 (B200 extension):
// BT sweeps of a star / box stencil fused into one pass over HBM.
//   level 0   input planes, TMA ring, extent (TA + 2 BT XR) x (TB + 2 BT R)
//   level s   sweep s over the tile grown by BT - s halos, two smem slots per level
//   level BT  the output tile, stored to HBM
// Every level runs the retimed scatter: 2R+1 rotating accumulators per point, one
// plane in, one completed plane out.  The pipeline is skewed — level s consumes the plane
// level s-1 emitted in the previous iteration — so one __syncthreads per plane orders all
// levels.  Points outside the interior keep their input value: the input halo is the
// boundary condition of every fused step (cst_sweep copies it into the output halo, so
// unfused ping-pong steps see the same values).  Intermediate planes never reach HBM.
// =============================================================================
constexpr int BT = CST_BT;
__host__ __device__ constexpr int tb_wa(int s) { return TA + 2 * XR * (BT - s); }
__host__ __device__ constexpr int tb_wb(int s) { return TB + 2 * R * (BT - s); }
__host__ __device__ constexpr int tb_nba(int s) { return tb_wa(s) / BMA; }
__host__ __device__ constexpr int tb_nblk(int s) { return tb_nba(s) * (tb_wb(s) / BMB); }
__host__ __device__ constexpr int tb_kb(int s) { return (tb_nblk(s) + NTHR - 1) / NTHR; }
constexpr int TB_NPB = BMA * BMB;  // points per register block
constexpr int TB_SLOT0 = round_slot(tb_wa(0) * tb_wb(0));
constexpr int TB_SLOTI = round_slot(tb_wa(1) * tb_wb(1));

template <int S>
struct TbAcc {
  double v[tb_kb(S) * TB_NPB][W];
  TbAcc<S + 1> next;
};
template <>
struct TbAcc<BT + 1> {};

template <int S, int L>
__device__ __forceinline__ auto& tb_acc(TbAcc<L>& a) {
  if constexpr (S == L) return a.v;
  else return tb_acc<S>(a.next);
}

// One level-S step of the skewed pipeline: plane q of level S-1 (src, row width
// tb_wa(S-1)) is scattered into the level-S accumulators; level-S plane q - R is then
// complete and goes to dst (level-S slot) or, for S == BT, to HBM.
template <int S, int U>
__device__ __forceinline__ void tb_stage(const Ctx& C, const cst_kparams& P, const SGeo& g,
                                         const double* __restrict__ src,
                                         double* __restrict__ dst,
                                         double (&acc)[tb_kb(S) * TB_NPB][W], int q) {
  constexpr int WA = tb_wa(S), SWA = tb_wa(S - 1);
  constexpr int NBA = tb_nba(S), NBLK = tb_nblk(S), KB = tb_kb(S);
  constexpr int HX = XR * (BT - S), HY = R * (BT - S);
  constexpr int WX = BMA + 2 * XR;   // x-window of a block row (src cols ex0 .. ex0 + WX)
  constexpr int ES = (U - R + W) % W;  // slot of the completed plane q - R
  // contribution d of plane q belongs to plane q - (d - R); only interior planes compute
  bool zin[W];
#pragma unroll
  for (int d = 0; d < W; ++d) {
    const int m = q - (d - R);
    zin[d] = m >= 0 && m < P.nz;
  }
  const int o = q - R;
#pragma unroll
  for (int kb = 0; kb < KB; ++kb) {
    const int blk = (int)threadIdx.x + kb * NTHR;
    if (KB * NTHR > NBLK && blk >= NBLK) continue;
    const int ex0 = (blk % NBA) * BMA, ey0 = (blk / NBA) * BMB;
    // level-S point (ex, ey) reads src at (ex + XR + dx, ey + R + dy)
    const double* base = src + ey0 * SWA + ex0;
    // contribution chains start from the accumulator they land in (no extra add);
    // points outside the interior restart from it below and keep their input value
    double c[BMB][BMA][W], ctr[BMB][BMA];
    auto accum = [&](int ib, int ia, int d) -> double& {
      return acc[kb * TB_NPB + ib * BMA + ia][(U - (d - R) + 2 * W) % W];
    };
    auto load_row = [&](int row, double* w) {
      if constexpr (BMA % 2 == 0) {
#pragma unroll
        for (int t = 0; t < WX / 2; ++t) {
          const double2 v = *reinterpret_cast<const double2*>(base + row * SWA + 2 * t);
          w[2 * t] = v.x;
          w[2 * t + 1] = v.y;
        }
      } else {
#pragma unroll
        for (int t = 0; t < WX; ++t) w[t] = base[row * SWA + t];
      }
    };
    if constexpr (KIND == 1) {
#pragma unroll
      for (int ib = 0; ib < BMB; ++ib) {
        double w[WX];
        load_row(R + ib, w);
#pragma unroll
        for (int ia = 0; ia < BMA; ++ia) {
          const double u0 = w[XR + ia];
          ctr[ib][ia] = u0;
          double ip = fma(C.coef(0), u0, accum(ib, ia, R));
#pragma unroll
          for (int k = -R; k <= R; ++k)
            if (k != 0) ip = fma(C.coef(star_ci(0, k)), w[XR + ia + k], ip);
          c[ib][ia][R] = ip;
#pragma unroll
          for (int d = 0; d < W; ++d)
            if (d != R) c[ib][ia][d] = fma(C.coef(star_ci(2, d - R)), u0, accum(ib, ia, d));
        }
      }
#pragma unroll
      for (int wr = -R; wr < BMB + R; ++wr) {  // y-neighbour rows of the block
        double v[BMA];
        if (wr >= 0 && wr < BMB) {
#pragma unroll
          for (int ia = 0; ia < BMA; ++ia) v[ia] = ctr[wr][ia];
        } else if constexpr (BMA % 2 == 0) {
#pragma unroll
          for (int ia = 0; ia < BMA; ia += 2) {
            const double2 t = *reinterpret_cast<const double2*>(base + (R + wr) * SWA + XR + ia);
            v[ia] = t.x;
            v[ia + 1] = t.y;
          }
        } else {
#pragma unroll
          for (int ia = 0; ia < BMA; ++ia) v[ia] = base[(R + wr) * SWA + XR + ia];
        }
#pragma unroll
        for (int ib = 0; ib < BMB; ++ib) {
          const int k = wr - ib;
          if (k == 0 || k < -R || k > R) continue;
#pragma unroll
          for (int ia = 0; ia < BMA; ++ia)
            c[ib][ia][R] = fma(C.coef(star_ci(1, k)), v[ia], c[ib][ia][R]);
        }
      }
    } else {  // box: slices dz of plane q, (dy, dx) ascending within each slice
#pragma unroll
      for (int ib = 0; ib < BMB; ++ib)
#pragma unroll
        for (int ia = 0; ia < BMA; ++ia)
#pragma unroll
          for (int d = 0; d < W; ++d) c[ib][ia][d] = accum(ib, ia, d);
#pragma unroll
      for (int wr = 0; wr < BMB + 2 * R; ++wr) {
        double w[WX];
        load_row(wr, w);
#pragma unroll
        for (int ib = 0; ib < BMB; ++ib) {
          const int dy = wr - R - ib;
          if (dy == 0) {
#pragma unroll
            for (int ia = 0; ia < BMA; ++ia) ctr[ib][ia] = w[XR + ia];
          }
          if (dy < -R || dy > R) continue;
#pragma unroll
          for (int ia = 0; ia < BMA; ++ia)
#pragma unroll
            for (int dx = -R; dx <= R; ++dx)
#pragma unroll
              for (int d = 0; d < W; ++d)
                c[ib][ia][d] = fma(C.coef(box_ci(d - R, dy, dx)), w[XR + ia + dx], c[ib][ia][d]);
        }
      }
    }
    // scatter into the rotating accumulators, emit plane q - R, clear its slot
#pragma unroll
    for (int ib = 0; ib < BMB; ++ib)
#pragma unroll
      for (int ia = 0; ia < BMA; ++ia) {
        double(&A)[W] = acc[kb * TB_NPB + ib * BMA + ia];
        const int gx = g.a0 - HX + ex0 + ia, gy = g.b0 - HY + ey0 + ib;
        const bool inxy = gx >= 0 && gx < P.nx && gy >= 0 && gy < P.ny;
#pragma unroll
        for (int d = 0; d < W; ++d) {
          const int sl = (U - (d - R) + 2 * W) % W;
          if (inxy && zin[d]) A[sl] = c[ib][ia][d];
          else if (d == R) A[sl] += ctr[ib][ia];  // outside: keep the input value
        }
        const double val = A[ES];
        A[ES] = 0.0;
        if constexpr (S < BT) {
          dst[(ey0 + ib) * WA + ex0 + ia] = val;
        } else {
          if (o >= g.s_start && o < g.s_end && gx < P.nx && gy < P.ny)
            put(P, 0, gx + (long long)gy * P.py + (long long)o * P.pz, val);
        }
      }
  }
}

template <int S, int L>
__device__ __forceinline__ void tb_zero(TbAcc<L>& a) {
  if constexpr (S <= BT) {
    auto& v = tb_acc<S>(a);
#pragma unroll
    for (int k = 0; k < tb_kb(S) * TB_NPB; ++k)
#pragma unroll
      for (int m = 0; m < W; ++m) v[k][m] = 0.0;
    tb_zero<S + 1>(a);
  }
}

template <int DUMMY>
__device__ __forceinline__ void kernel_tblock(const cst_kparams& P, double* smem) {
  Ctx C{P};
  constexpr int D = PF, NP = PF;
  constexpr unsigned BYTES0 = (unsigned)(tb_wa(0) * tb_wb(0) * 8);
  const SGeo g = stream_geo(P);
  const int tid = threadIdx.x;
  const int n_load = (g.s_end - g.s_start) + 2 * BT * R;  // input planes of this chunk
  const int n_it = n_load + BT - 1;                       // + pipeline skew
  const int p0 = g.s_start - BT * R;
  double* lvl = smem + NP * TB_SLOT0;  // level s slot t at lvl + ((s-1)*2 + t) * TB_SLOTI
  u64* bars = (u64*)(lvl + (BT - 1) * 2 * TB_SLOTI);
  TbAcc<1> acc;
  tb_zero<1>(acc);
  if (tid == 0) {
    for (int s = 0; s < NP; ++s) mbar_init(&bars[s], 1);
    fence_mbar_init();
  }
  __syncthreads();
  auto issue = [&](int j) {  // input plane p0 + j -> ring slot j % NP
    const int sl = j % NP;
    mbar_arrive_expect_tx(&bars[sl], BYTES0);
    tma_load_3d(smem + sl * TB_SLOT0, &P.tma[0], &bars[sl], P.tox + g.a0 - XR * BT,
                P.toy + g.b0 - R * BT, P.toz + p0 + j);
  };
  if (tid == 0)
    for (int j = 0; j < D && j < n_load; ++j) issue(j);

  for (int i0 = 0; i0 < n_it; i0 += W) {
    static_for<0, W>([&](auto UU) {
      constexpr int u = decltype(UU)::value;
      const int i = i0 + u;
      if (i >= n_it) return;  // CTA-uniform
      const int p = p0 + i;
      // levels BT..2 consume last iteration's planes while the TMA of plane p lands
      static_for<2, BT + 1>([&](auto SS) {
        constexpr int S = BT + 2 - decltype(SS)::value;
        const double* src = lvl + ((S - 2) * 2 + ((i - 1) & 1)) * TB_SLOTI;
        double* dst = S < BT ? lvl + ((S - 1) * 2 + (i & 1)) * TB_SLOTI : nullptr;
        tb_stage<S, u>(C, P, g, src, dst, tb_acc<S>(acc), p - (S - 1) * (R + 1));
      });
      if (i < n_load) {
        mbar_wait(&bars[i % NP], (u32)((i / NP) & 1));
        tb_stage<1, u>(C, P, g, smem + (i % NP) * TB_SLOT0, lvl + (i & 1) * TB_SLOTI,
                       tb_acc<1>(acc), p);
      }
      __syncthreads();
      if (tid == 0 && i + D < n_load) {
        fence_proxy_async();
        issue(i + D);
      }
    });
  }
}


// In-plane part of the star in row-scatter form: the block's window rows are visited
// once, top to bottom, and each row's values are added into the in-plane sums of the block
// rows within R (y-terms) — plus, for the block's own rows, the x-terms and the centre.
// Only the block's sums, centres and one row window are live: the register budget of the
// TMEM path, whose streamed state is not in registers.
template <class LD>
__device__ __forceinline__ void star_inplane_rows(const Ctx& C, const LD& ld, const int* la,
                                                  const int* lb, double (&ip)[NCB][NCA],
                                                  double (&cen)[NCB][NCA]) {
#pragma unroll
  for (int cb = 0; cb < CMB; ++cb) {
    const int lb0 = lb[cb * BMB];
#pragma unroll
    for (int ca = 0; ca < CMA; ++ca) {
      const int la0 = la[ca * BMA];
#pragma unroll
      for (int wr = -R; wr < BMB + R; ++wr) {
        if (wr >= 0 && wr < BMB) {
          double w[BMA + 2 * XR];
          load_xwin(ld, la0, lb0 + wr, w);
#pragma unroll
          for (int b = 0; b < BMA; ++b) {
            const double c = w[XR + b];
            double x = C.coef(0) * c;
#pragma unroll
            for (int k = -R; k <= R; ++k)
              if (k != 0) x = fma(C.coef(star_ci(AX_A, k)), w[XR + b + k], x);
            // every sum was started by its k = -R row (visited first), so add here
            ip[cb * BMB + wr][ca * BMA + b] += x;
            cen[cb * BMB + wr][ca * BMA + b] = c;
#pragma unroll
            for (int rb = 0; rb < BMB; ++rb) {
              const int k = wr - rb;
              if (k == 0 || k < -R || k > R) continue;
              double& B = ip[cb * BMB + rb][ca * BMA + b];
              B = (k == -R) ? C.coef(star_ci(AX_B, k)) * c : fma(C.coef(star_ci(AX_B, k)), c, B);
            }
          }
        } else {
          double v[BMA];
          if constexpr (LD::VEC && (BMA % 2 == 0)) {
#pragma unroll
            for (int b = 0; b < BMA; b += 2) {
              const double2 t = ld.at2(la0 + b, lb0 + wr);
              v[b] = t.x;
              v[b + 1] = t.y;
            }
          } else {
#pragma unroll
            for (int b = 0; b < BMA; ++b) v[b] = ld.at(la0 + b, lb0 + wr);
          }
#pragma unroll
          for (int b = 0; b < BMA; ++b)
#pragma unroll
            for (int rb = 0; rb < BMB; ++rb) {
              const int k = wr - rb;
              if (k < -R || k > R) continue;
              double& B = ip[cb * BMB + rb][ca * BMA + b];
              B = (k == -R) ? C.coef(star_ci(AX_B, k)) * v[b] : fma(C.coef(star_ci(AX_B, k)), v[b], B);
            }
        }
      }
    }
  }
}

// =============================================================================
// star, streamed-direction state in tensor memory (qstore = 2)
//
// The retimed star keeps 2R+1 pending outputs per point in registers, which caps the
// register blocking (merging) and so the shared-memory reuse of the in-plane
// windows: at BM 2x2 the x/y windows cost ~10 smem loads per point and the kernel is
// bound by the shared-memory pipe (profiles/).  Here the per-point streamed state lives in
// TMEM instead — a ring of R (u, A) pairs per point, where at plane q
//   A(q)     = ip(q) + sum_{k=-R..-1} ws[k] u(q+k)          (in-plane part + lower half)
//   out(q-R) = A(q-R) + sum_{k=1..R-1} ws[k] u(q-R+k) + ws[R] u(q)
// (the retimed split of P:69: each plane's contributions are added once, in plane order)
// — so the registers hold only the current plane and the block can grow to 4x4 points.
// TMEM reads run beside the shared-memory pipe (tools/tmem_bench.cu).
// Layout: warp w -> lanes 32*(w%4) + lane, column block (w/4) * NPT*4R; point i of the
// thread at +i*4R: u slots [0, 2R), A slots [2R, 4R), slot s = plane index mod R.
// =============================================================================
constexpr int NPT = NCA * NCB;
constexpr int TM_WPQ = (NTHR / 32 + 3) / 4;  // warps sharing one TMEM lane quarter
// columns per point: star R (u, A) pairs; hypterm R slots of E_0..4 and R of A_0..4
constexpr int TM_PCOLS = KIND == 3 ? 20 * R : 4 * R;
constexpr int TM_USED = TM_WPQ * NPT * TM_PCOLS;
constexpr int TM_COLS = TM_USED <= 32 ? 32 : TM_USED <= 64 ? 64 : TM_USED <= 128 ? 128
                      : TM_USED <= 256 ? 256 : 512;

template <int DUMMY>
__device__ __forceinline__ void kernel_star_tmem(const cst_kparams& P, double* smem) {
  static_assert(DUMMY != 0 || (KIND == 1 && STAGING == 3 && TS == 1),
                "TMEM queue: star, TMA, T_SD = 1");
  static_assert(DUMMY != 0 || TM_USED <= 512, "TMEM queue exceeds 512 columns");
  Ctx C{P};
  constexpr int D = PF, NP = PF;
  const int ta = thread_x();
  const int tb = SZ ? thread_y() : thread_z();
  const int tid = threadIdx.x, warp = tid / 32;
  double* __restrict__ out = P.out[0];
  u64* bars = (u64*)(smem + NP * SLOT);
  u32* tslot = (u32*)(bars + NP);  // spare mbarrier words (kernel_smem_bytes reserves 2 NP)

  int la[NCA], lb[NCB];
#pragma unroll
  for (int i = 0; i < NCA; ++i) la[i] = merged_pos(i, ta, TBA, BMA);
#pragma unroll
  for (int i = 0; i < NCB; ++i) lb[i] = merged_pos(i, tb, TBB, BMB);

  if (warp == 0) tmem_alloc(tslot, TM_COLS);
  if (tid == 0) {
    for (int s = 0; s < NP; ++s) mbar_init(&bars[s], 1);
    fence_mbar_init();
  }
  tmem_fence_before_sync();
  __syncthreads();
  tmem_fence_after_sync();
  const u32 tq = *tslot + ((u32)((warp & 3) * 32) << 16) + (u32)((warp >> 2) * NPT * TM_PCOLS);
  auto ws = [&](int k) { return C.coef(star_ci(AX_S, k)); };
  const SGeo g = stream_geo(P);
  const int n_planes = (g.s_end - g.s_start) + 2 * R;
  const long long col0 = (long long)g.a0 + (long long)g.b0 * g.st_b;
  if (tid == 0) {
    for (int j = 0; j < D && j < n_planes; ++j) {
      const int sl = j % NP;
      mbar_arrive_expect_tx(&bars[sl], PL * 8);
      tma_plane(P, g, smem + sl * SLOT, &bars[sl], g.s_start - R + j);
    }
  }

  // one plane per iteration, ring slots rotated at run time (slot of plane j = j mod R):
  // a compile-time rotation would need R unrolled copies of the plane, whose hoisted
  // invariants cost more registers than the TMEM ring saves
#pragma unroll 1
  for (int j = 0; j < n_planes; ++j) {
    const int p = g.s_start - R + j;
    const int slot = j % NP;
    const int u = j % R;
    mbar_wait(&bars[slot], (u32)((j / NP) & 1));
    const SmemPlane ld{smem + slot * SLOT};
    const bool need_a = j >= R && j < n_planes - R;  // A(p) feeds an interior output
    u32 cu[R];  // column of u(p - R + m), m = 0..R-1: slot (j + m) mod R
#pragma unroll
    for (int m = 0; m < R; ++m) cu[m] = (u32)(2 * ((u + m) % R));
    const u32 cs = (u32)(2 * u);  // this plane's slot (holds plane j - R until rewritten)
    auto issue = [&](int pt, TmQ<R>& q) {
      const u32 tp = tq + (u32)(pt * TM_PCOLS);
      u32 ta[R];
#pragma unroll
      for (int m = 0; m < R; ++m) ta[m] = tp + cu[m];
      tmem_ld_issue<R>(ta, tp + 2 * R + cs, q);
    };
    // TMEM loads in flight while the in-plane part is computed: every point's ring when
    // they fit the register budget (TM_ALL), else point 0's, then point pt + 1's while
    // point pt is finished (one-deep pipeline)
    constexpr bool TM_ALL = NPT * (2 * R + 2) <= 48;
    TmQ<R> qa[TM_ALL ? NPT : 2];
    if (j >= R) {
      if constexpr (TM_ALL) static_for<0, NPT>([&](auto PP) { issue(decltype(PP)::value, qa[decltype(PP)::value]); });
      else issue(0, qa[0]);
    }
    double ip[NCB][NCA], cen[NCB][NCA];
    if (need_a) star_inplane_rows(C, ld, la, lb, ip, cen);
    else load_centres(ld, la, lb, cen);
    if constexpr (TM_ALL) {
      if (j >= R) {
        tmem_wait_ld();
        static_for<0, NPT>([&](auto PP) { tmem_pin(qa[decltype(PP)::value].r); });
      }
    }
    auto finish = [&](auto PP, TmQ<R>& q, TmQ<R>& qn) {
      constexpr int pt = decltype(PP)::value, ib = pt / NCA, ia = pt % NCA;
      const u32 tp = tq + (u32)(pt * TM_PCOLS);
      if (j >= R) {
        if constexpr (!TM_ALL) {
          tmem_ld_wait<R>(q);
          if constexpr (pt + 1 < NPT) issue(pt + 1, qn);
        }
        if (need_a) {  // A(p) = ip(p) + sum_{k=-R..-1} ws[k] u(p+k)
          double a = ip[ib][ia];
#pragma unroll
          for (int m = 0; m < R; ++m) a = fma(ws(m - R), tmq_u<R>(q, m), a);
          tmem_st_d(tp + 2 * R + cs, a);
        }
        if (j >= 2 * R) {  // out(p-R) = A(p-R) + sum_{k=1..R-1} ws[k] u(p-R+k) + ws[R] u(p)
          double o = tmq_a<R>(q);
#pragma unroll
          for (int k = 1; k < R; ++k) o = fma(ws(k), tmq_u<R>(q, k), o);
          o = fma(ws(R), cen[ib][ia], o);
          if (g.a0 + la[ia] < g.n_a && g.b0 + lb[ib] < g.n_b) {
            const long long off =
                col0 + la[ia] + (long long)lb[ib] * g.st_b + (long long)(p - R) * g.st_s;
            out[off] = o;
            if constexpr (CST_REMOTE) P.rout[0][off] = o;
          }
        }
      }
      tmem_st_d(tp + cs, cen[ib][ia]);
    };
    static_for<0, NPT>([&](auto PP) {
      constexpr int pt = decltype(PP)::value;
      if constexpr (TM_ALL) finish(PP, qa[pt], qa[pt]);
      else if constexpr (pt % 2 == 0) finish(PP, qa[0], qa[1]);
      else finish(PP, qa[1], qa[0]);
    });
    tmem_wait_st();  // the next plane reads these slots
    __syncthreads();
    if (tid == 0 && j + D < n_planes) {
      const int sl = (j + D) % NP;
      fence_proxy_async();
      mbar_arrive_expect_tx(&bars[sl], PL * 8);
      tma_plane(P, g, smem + sl * SLOT, &bars[sl], p + D);
    }
  }
  tmem_fence_before_sync();
  __syncthreads();
  tmem_fence_after_sync();
  if (warp == 0) tmem_dealloc(*tslot, TM_COLS);
}


// =============================================================================
// hypterm in-plane terms by row streaming (TMEM path, one point per thread)
//
// Every in-plane derivative contributes  sum_{k=-R..R, k!=0} wd[k] E^d_f(p + k e_d)  to flux f,
// wd[k] = -sign(k) dxinv_d a_|k| (the bank's ws tables, one per direction), E^d_f the
// pointwise products of direction d.  Instead of loading a window per array and point, the
// lanes walk the union of their windows one position at a time:
//  * along a (x): the products E^a_f are formed once per column into shared-memory product
//    planes (hyp_prod_a, round 2; round 1 walked six inputs per position and formed the
//    products per lane); lanes 2i, 2i+1 share each 16-B chunk of the 2R+2 positions starting
//    at the even element la - XR - (la & 1); a lane's weight at position j is
//    wd[j - XR - (la & 1)], chosen by a select between two uniform constants;
//  * along b each lane walks its own 2R rows (six loads, five products, five FMAs per row;
//    with two points stacked along b, the union of their rows).  (CST_HYP_HPAIR = 1, experiment: when a warp
//    holds two b-rows (T_a = 16) both half-warps read the same row at a time, 2R+2 rows per
//    pair, the weight selected by the row parity — measured slower: 3.85 vs 3.53 ms at
//    512^3; the shared 8-byte loads of the two half-warps are not merged into one wavefront.)
// Positions outside a lane's window (beyond its halo) are predicated off, never weighted by
// zero, so halo garbage past the radius cannot leak in as 0 * NaN.
// =============================================================================
#ifndef CST_HYP_HPAIR
#define CST_HYP_HPAIR 0
#endif
constexpr bool HPAIR = CST_HYP_HPAIR && TBA == 16 && TBB % 2 == 0;  // two b-rows per warp
#ifndef CST_HYP_WXPRE
#define CST_HYP_WXPRE 1  // TMEM hypterm: per-lane x weights selected once per thread
#endif
#ifndef CST_TM_EARLY
#define CST_TM_EARLY (CST_BMX * CST_BMY * CST_BMZ > 1)  // TMEM hypterm: ring fetch before in-plane
#endif
constexpr bool TM_EARLY = CST_TM_EARLY;


// E^d_f at one position from v = {cons1..4, q_d, q4}
template <int DIR>
__device__ __forceinline__ void hyp_e(const double (&v)[6], double (&E)[5]) {
  E[0] = v[DIR];
#pragma unroll
  for (int m = 0; m < 3; ++m) E[m + 1] = m == DIR ? fma(v[m], v[4], v[5]) : v[m] * v[4];
  E[4] = fma(v[3], v[4], v[5] * v[4]);
}

// A_f += w E_f with the lane's weight for offsets k0 (parity 0) / k1 (parity 1)
template <int DIR, int K0, int K1>
__device__ __forceinline__ void hyp_acc(const Ctx& C, bool par, const double (&E)[5],
                                        double (&A)[5]) {
  constexpr bool V0 = K0 != 0 && K0 >= -R && K0 <= R, V1 = K1 != 0 && K1 >= -R && K1 <= R;
  if constexpr (V0 && V1) {  // K1 = K0 - 1: both on the same side of 0, same sign
    static_assert((K0 > 0) == (K1 > 0), "weights of one sign");
    constexpr int I0 = ws_base(DIR) + (K0 < 0 ? -K0 : K0) - 1;
    constexpr int I1 = ws_base(DIR) + (K1 < 0 ? -K1 : K1) - 1;
    const double p = par ? C.coef(I1) : C.coef(I0);
    const double w = K0 > 0 ? -p : p;
#pragma unroll
    for (int f = 0; f < 5; ++f) A[f] = fma(w, E[f], A[f]);
  } else if constexpr (V0) {
    if (!par) {
#pragma unroll
      for (int f = 0; f < 5; ++f) A[f] = fma(hws(C, DIR, K0), E[f], A[f]);
    }
  } else if constexpr (V1) {
    if (par) {
#pragma unroll
      for (int f = 0; f < 5; ++f) A[f] = fma(hws(C, DIR, K1), E[f], A[f]);
    }
  }
}

// the lane's x weights at the walk positions where both parities have one (positions
// 1..R-1 and R+2..2R: w = -sign(k) P_x[|k|] with k = j - XR - parity), selected once per
// thread (CST_HYP_WXPRE) instead of once per position and plane
struct HypWx {
  double w[2 * R - 2 > 0 ? 2 * R - 2 : 1];
};
__device__ __forceinline__ HypWx hyp_wx(const Ctx& C, bool odd) {
  HypWx W;
  int n = 0;
#pragma unroll
  for (int j = 0; j < 2 * R + 2; ++j) {
    const int k0 = j - XR, k1 = j - XR - 1;
    const bool v0 = k0 != 0 && k0 >= -R && k0 <= R, v1 = k1 != 0 && k1 >= -R && k1 <= R;
    if (v0 && v1) W.w[n++] = odd ? hws(C, DA, k1) : hws(C, DA, k0);
  }
  return W;
}
constexpr int hyp_wx_slot(int j) {  // index into HypWx::w of walk position j, -1 if none
  int n = 0;
  for (int i = 0; i < j; ++i) {
    const int k0 = i - XR, k1 = i - XR - 1;
    if (k0 != 0 && k0 >= -R && k0 <= R && k1 != 0 && k1 >= -R && k1 <= R) ++n;
  }
  const int k0 = j - XR, k1 = j - XR - 1;
  return (k0 != 0 && k0 >= -R && k0 <= R && k1 != 0 && k1 >= -R && k1 <= R) ? n : -1;
}

// b-direction terms into A
template <class LD>
__device__ __forceinline__ void hyp_rows_b(const Ctx& C, const LD* ld, int la, int lb,
                                           double (&A)[5]) {
  if constexpr (HPAIR) {
    const bool odd = lb & 1;
    const int b0 = lb - (int)odd - R;
    static_for<0, 2 * R + 2>([&](auto QQ) {
      constexpr int q = decltype(QQ)::value;
      double v[6];
#pragma unroll
      for (int m = 0; m < 4; ++m) v[m] = ld[m].at(la, b0 + q);
      v[4] = ld[Q_B].at(la, b0 + q);
      v[5] = ld[7].at(la, b0 + q);
      double E[5];
      hyp_e<DB>(v, E);
      hyp_acc<DB, q - R, q - R - 1>(C, odd, E, A);
    });
  } else {
    static_for<0, 2 * R + 1>([&](auto QQ) {
      constexpr int q = decltype(QQ)::value;
      if constexpr (q != R) {
        double v[6];
#pragma unroll
        for (int m = 0; m < 4; ++m) v[m] = ld[m].at(la, lb - R + q);
        v[4] = ld[Q_B].at(la, lb - R + q);
        v[5] = ld[7].at(la, lb - R + q);
        double E[5];
        hyp_e<DB>(v, E);
        hyp_acc<DB, q - R, q - R>(C, false, E, A);
      }
    });
  }
}

// b-direction terms of NP2 points stacked along b (rows lb0 .. lb0 + NP2 - 1, register
// blocking BM_b): the union of their windows is walked once, each row's products
// feeding every point it neighbours (2R + NP2 rows instead of 2R per point)
template <int NP2, class LD>
__device__ __forceinline__ void hyp_rows_bn(const Ctx& C, const LD* ld, int la, int lb0,
                                            double (&A)[NP2][5]) {
  static_for<0, 2 * R + NP2>([&](auto QQ) {
    constexpr int q = decltype(QQ)::value;
    if constexpr (NP2 > 1 || q != R) {
      double v[6];
#pragma unroll
      for (int m = 0; m < 4; ++m) v[m] = ld[m].at(la, lb0 - R + q);
      v[4] = ld[Q_B].at(la, lb0 - R + q);
      v[5] = ld[7].at(la, lb0 - R + q);
      double E[5];
      hyp_e<DB>(v, E);
      static_for<0, NP2>([&](auto PP) {
        constexpr int pt = decltype(PP)::value;
        hyp_acc<DB, q - R - pt, q - R - pt>(C, false, E, A[pt]);
      });
    }
  });
}

// =============================================================================
// hypterm-like, streamed-direction state in tensor memory (qstore = 2)
//
// The retimed hypterm kernel keeps 5 fluxes x (2R+1) pending planes = 45 doubles per point
// in registers (202-244 registers, 8 warps per SM, latency-bound: profiles/).  Here the
// state is a TMEM ring per point: R slots of the streamed-direction products E_f and R
// slots of the partial fluxes A_f, with, at plane q (the retimed split of P:69),
//   A_f(q)      = -T_a,f(q) - T_b,f(q) + sum_{k=-R..-1} ws[k] E_f(q+k)
//   flux_f(q-R) = A_f(q-R) + sum_{k=1..R-1} ws[k] E_f(q-R+k) + ws[R] E_f(q)
// Both sums read the same ring slots (planes q-R .. q-1), fetched while the in-plane
// terms T are computed from shared memory (T_a from the x-product planes below, T_b by the
// b row walk).  Slot of plane j = j mod R, rotated at run time.
// Layout per point (20R columns): E slot s at 10 s, A slot s at 10 (R + s); 5 doubles each.
// =============================================================================
// x-direction product planes (the TMEM hypterm path, round 2): E^a_f of every column of the
// tile and its x-halo is formed once per plane (own columns by their threads, the 2 XR halo
// columns by spare threads) into a double-buffered shared-memory plane; the x-derivative then
// reads 5 products per position instead of forming them from 6 inputs (the round-1 x row
// walk formed each product 2R times, once per point whose window holds it): 3.19 vs 3.27 ms
// at 512^3 (4 interleaved rounds, profiles/r02/g34), 2 prefetch stages (the planes take the
// smem of the third).  Per plane: own loads, E^x and E^s, halo E^x, b-walk -> CTA barrier
// (products visible, ring slot read) -> TMA refill -> D_x from the planes -> TMEM ring.
constexpr bool XPROD = KIND == 3 && QTM;
constexpr int XP_PITCH = TA + 2 * XR;                 // row pitch of a product plane
constexpr int XP_SLOT = round_slot(XP_PITCH * TB);    // one product plane (elements)
constexpr int XP_BUF = XPROD ? 2 * 5 * XP_SLOT : 0;  // two buffers of 5 products
// D_a of the 5 fluxes from the product planes at (la, lb) into A (same weights and walk
// as the round-1 x row walk: lanes 2i, 2i+1 share each 16-B chunk of the 2R+2 positions)
__device__ __forceinline__ void hyp_prod_a(const Ctx& C, const double* pb, int la, int lb,
                                           double (&A)[5], const HypWx* wx) {
  const bool odd = la & 1;
  const int e0 = la - XR - (int)odd;  // tile-local x of the first walk position
  const double* row = pb + lb * XP_PITCH + XR + e0;
  static_for<0, R + 1>([&](auto CC) {
    constexpr int c = decltype(CC)::value;
    double2 v2[5];
#pragma unroll
    for (int f = 0; f < 5; ++f)
      v2[f] = *reinterpret_cast<const double2*>(row + f * XP_SLOT + 2 * c);
    static_for<0, 2>([&](auto HH) {
      constexpr int h = decltype(HH)::value, j = 2 * c + h;
      double E[5];
#pragma unroll
      for (int f = 0; f < 5; ++f) E[f] = h ? v2[f].y : v2[f].x;
      constexpr int ws_i = hyp_wx_slot(j);
      if (ws_i >= 0 && wx != nullptr) {
#pragma unroll
        for (int f = 0; f < 5; ++f) A[f] = fma(wx->w[ws_i < 0 ? 0 : ws_i], E[f], A[f]);
      } else {
        hyp_acc<DA, j - XR, j - XR - 1>(C, odd, E, A);
      }
    });
  });
}

template <int DUMMY>
__device__ __forceinline__ void kernel_hyp_tmem(const cst_kparams& P, double* smem) {
  static_assert(DUMMY != 0 || (KIND == 3 && STAGING == 3 && TS == 1 && NCA == 1 && CMB == 1 &&
                               NCB <= 2),
                "TMEM hypterm: TMA, T_SD = 1, one point along a, up to two along b");
  static_assert(DUMMY != 0 || TM_USED <= 512, "TMEM ring exceeds 512 columns");
  Ctx C{P};
  constexpr int D = PF, NP = PF;
  const SGeo g = stream_geo(P);
  const int ta = thread_x();
  const int tb = SZ ? thread_y() : thread_z();
  const int tid = threadIdx.x, warp = tid / 32;
  const int n_planes = (g.s_end - g.s_start) + 2 * R;
  double* pbuf = smem + NP * RSLOT;  // x-product planes (XPROD), 2 x 5 x XP_SLOT
  u64* bars = (u64*)(smem + NP * RSLOT + XP_BUF);
  u32* tslot = (u32*)(bars + NP);  // spare mbarrier words (kernel_smem_bytes reserves 2 NP)

  int la[NCA], lb[NCB];
#pragma unroll
  for (int i = 0; i < NCA; ++i) la[i] = merged_pos(i, ta, TBA, BMA);
#pragma unroll
  for (int i = 0; i < NCB; ++i) lb[i] = merged_pos(i, tb, TBB, BMB);
  const long long col0 = (long long)g.a0 + (long long)g.b0 * g.st_b;
  // streamed-direction weights (as kernel_hyp_stream1): plane p adds ws[p-o] E_f(p) to o
  auto ws = [&](int k) { return hws(C, DS, k); };

  if (warp == 0) tmem_alloc(tslot, TM_COLS);
  if (tid == 0) {
    for (int s = 0; s < NP; ++s) mbar_init(&bars[s], 1);
    fence_mbar_init();
  }
  tmem_fence_before_sync();
  __syncthreads();
  tmem_fence_after_sync();
  const u32 tq = *tslot + ((u32)((warp & 3) * 32) << 16) + (u32)((warp >> 2) * NPT * TM_PCOLS);
  const HypWx wxl = hyp_wx(C, la[0] & 1);
  if (tid == 0)
    for (int j = 0; j < D && j < n_planes; ++j) {
      mbar_arrive_expect_tx(&bars[j % NP], TX_BYTES);
      tma_plane(P, g, smem + (j % NP) * RSLOT, &bars[j % NP], g.s_start - R + j);
    }

#pragma unroll 1
  for (int j = 0; j < n_planes; ++j) {
    const int p = g.s_start - R + j;
    const int slot = j % NP;
    const int u = j % R;
    mbar_wait(&bars[slot], (u32)((j / NP) & 1));
    SPlane ld[NIN];
#pragma unroll
    for (int a = 0; a < NIN; ++a) ld[a] = splane(smem + slot * RSLOT, a);
    const bool need_a = j >= R && j < n_planes - R;  // A(p) feeds an interior output
    u32 ce[R];  // column offset of E slot of plane p - R + m
#pragma unroll
    for (int m = 0; m < R; ++m) ce[m] = (u32)(10 * ((u + m) % R));
    const u32 ca = (u32)(10 * (R + u));  // A slot of plane p - R (read) / p (written)
    {  // NCB points stacked along b (R15: BM_a = CM = 1, BM_b <= 2)
      constexpr int ia = 0;
      double E[NCB][5];
      double A[NCB][5];
      // ring slots of every point; with two points the CTA is TMEM-bound to 8 warps per SM
      // and registers are plentiful, so the rings are fetched before the in-plane terms
      // (load latency hidden by them); one point: fetched after them (fewer live registers)
      constexpr bool EARLY = TM_EARLY;
      u32 re[NCB][R][10], ra[NCB][10];
      auto issue_ring = [&](int ib) {
        const u32 tp = tq + (u32)(ib * TM_PCOLS);
#pragma unroll
        for (int m = 0; m < R; ++m) {
          tmem_ld_x8(tp + ce[m], re[ib][m]);
          tmem_ld_x2(tp + ce[m] + 8, re[ib][m] + 8);
        }
        tmem_ld_x8(tp + ca, ra[ib]);
        tmem_ld_x2(tp + ca + 8, ra[ib] + 8);
      };
      if (EARLY && j >= R) {
#pragma unroll
        for (int ib = 0; ib < NCB; ++ib) issue_ring(ib);
      }
      {
        static_assert(DUMMY != 0 || XPROD, "TMEM hypterm: x-product planes");
        // own columns: centres and E^a into the product planes of this plane's buffer; the
        // x-halo columns' E^a by the first 2 XR * TB threads; the b-terms; E^s.  Then the CTA
        // barrier (products visible, ring slot read), the refill, and D_a from the products.
        double* pb = pbuf + (j & 1) * 5 * XP_SLOT;
        double cen[NCB][5];
        double Ab[NCB][5];
#pragma unroll
        for (int ib = 0; ib < NCB; ++ib) {
#pragma unroll
          for (int m = 0; m < 4; ++m) cen[ib][m] = ld[m].at(la[0], lb[ib]);
          cen[ib][4] = ld[7].at(la[0], lb[ib]);
          const double qs = ld[4 + DS].at(la[0], lb[ib]);
          if (need_a) {
            const double v[6] = {cen[ib][0], cen[ib][1], cen[ib][2], cen[ib][3],
                                 ld[Q_A].at(la[0], lb[ib]), cen[ib][4]};
            double Ea[5];
            hyp_e<DA>(v, Ea);
#pragma unroll
            for (int f = 0; f < 5; ++f) pb[f * XP_SLOT + lb[ib] * XP_PITCH + XR + la[0]] = Ea[f];
          }
          const double vs[6] = {cen[ib][0], cen[ib][1], cen[ib][2], cen[ib][3], qs, cen[ib][4]};
          hyp_e<DS>(vs, E[ib]);
        }
        if (need_a) {
          // x-halo columns of the product planes, one thread per column (splitting each
          // column's products over two threads measured slower: 3.146 vs 3.105 ms, g38)
          for (int e = tid; e < 2 * XR * TB; e += NTHR) {
            const int hc = e % (2 * XR), hr = e / (2 * XR);
            const int hx = hc < XR ? hc - XR : TA + hc - XR;  // tile-local x of the column
            double v[6];
#pragma unroll
            for (int m = 0; m < 4; ++m) v[m] = ld[m].at(hx, hr);
            v[4] = ld[Q_A].at(hx, hr);
            v[5] = ld[7].at(hx, hr);
            double Ea[5];
            hyp_e<DA>(v, Ea);
#pragma unroll
            for (int f = 0; f < 5; ++f) pb[f * XP_SLOT + hr * XP_PITCH + XR + hx] = Ea[f];
          }
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib)
#pragma unroll
            for (int f = 0; f < 5; ++f) A[ib][f] = Ab[ib][f] = 0.0;
          if constexpr (NCB == 1 && HPAIR)
            hyp_rows_b(C, ld, la[0], lb[0], Ab[0]);
          else
            hyp_rows_bn<NCB>(C, ld, la[0], lb[0], Ab);
        }
        __syncthreads();
        if (tid == 0 && j + D < n_planes) {
          const int sl = (j + D) % NP;
          fence_proxy_async();
          mbar_arrive_expect_tx(&bars[sl], TX_BYTES);
          tma_plane(P, g, smem + sl * RSLOT, &bars[sl], p + D);
        }
        if (need_a) {
#pragma unroll
          for (int ib = 0; ib < NCB; ++ib) {
            hyp_prod_a(C, pb, la[0], lb[ib], A[ib], CST_HYP_WXPRE ? &wxl : nullptr);
#pragma unroll
            for (int f = 0; f < 5; ++f) A[ib][f] += Ab[ib][f];
          }
        }
      }
      // streamed-direction state, one point at a time (ring loaded after the in-plane terms)
#pragma unroll
      for (int ib = 0; ib < NCB; ++ib) {
        const u32 tp = tq + (u32)(ib * TM_PCOLS);
        if (j >= R) {
          if (!EARLY) issue_ring(ib);
          if (!EARLY || ib == 0) tmem_wait_ld();
#pragma unroll
          for (int m = 0; m < R; ++m) tmem_pin(re[ib][m]);
          tmem_pin(ra[ib]);
          auto ev = [&](int m, int f) { return tmem_d(re[ib][m][2 * f], re[ib][m][2 * f + 1]); };
          if (need_a) {
#pragma unroll
            for (int f = 0; f < 5; ++f)
#pragma unroll
              for (int m = 0; m < R; ++m) A[ib][f] = fma(ws(m - R), ev(m, f), A[ib][f]);
            tmem_st_5d(tp + ca, A[ib]);
          }
          if (j >= 2 * R) {
            double v[5];
#pragma unroll
            for (int f = 0; f < 5; ++f) {
              double o = tmem_d(ra[ib][2 * f], ra[ib][2 * f + 1]);
#pragma unroll
              for (int k = 1; k < R; ++k) o = fma(ws(k), ev(k, f), o);
              v[f] = fma(ws(R), E[ib][f], o);
            }
            if (g.a0 + la[ia] < g.n_a && g.b0 + lb[ib] < g.n_b) {
              const long long off =
                  col0 + la[ia] + (long long)lb[ib] * g.st_b + (long long)(p - R) * g.st_s;
#pragma unroll
              for (int f = 0; f < 5; ++f) put(P, f, off, v[f]);
            }
          }
        }
        tmem_st_5d(tp + 10 * u, E[ib]);
      }
    }
#if !CST_HYP_ROWS
#error "CST_HYP_ROWS = 0 (window path) was removed from the TMEM hypterm kernel"
#endif
    tmem_wait_st();  // the next plane reads these slots (waiting at the next plane's ring
                     // fetch instead measured the same: 3.171 vs 3.170 ms, g25)
    // (the plane's CTA barrier and ring refill are mid-plane, after the product planes)
  }
  tmem_fence_before_sync();
  __syncthreads();
  tmem_fence_after_sync();
  if (warp == 0) tmem_dealloc(*tslot, TM_COLS);
}

// =============================================================================
// entry point
// =============================================================================
// TMEM path: cap the registers at ~96 + 4 per point of the block (minimum resident CTAs
// for ptxas) — with the ring in TMEM the registers only hold the current plane, and the
// unconstrained schedule hoists every shared-memory load of the block (up to 255 registers)
#define CST_TM_NPT (CST_BMX * CST_CMX * CST_BMY * CST_CMY * CST_BMZ * CST_CMZ)
#define CST_TM_NTHR (CST_TBX * CST_TBY * CST_TBZ)
#if CST_KIND == 3
#define CST_TM_REGS (CST_TM_NPT == 1 ? 120 : 255)  // hypterm (two points: TMEM-bound to 8 warps/SM)
#else  // star: + every point's ring in flight when it fits 48 registers (TM_ALL)
#define CST_TM_REGS (96 + 4 * CST_TM_NPT + \
                     (CST_TM_NPT * (2 * CST_R + 2) <= 48 ? CST_TM_NPT * (2 * CST_R + 2) : 0))
#endif
#ifndef CST_TM_MINB
#define CST_TM_MINB (65536 / (CST_TM_NTHR * CST_TM_REGS) > 0 ? 65536 / (CST_TM_NTHR * CST_TM_REGS) : 1)
#endif
#if CST_QSTORE == 2 && CST_KIND != 4
#define CST_LB __launch_bounds__(CST_TBX * CST_TBY * CST_TBZ, CST_TM_MINB)
#elif CST_KIND == 4 && CST_RET == 2 && CST_BMX == 1
// rhs4 retimed, one point per thread: cap at ~168 registers (3 CTAs of 128 threads: 1.05 vs
// 1.22 ms at 216 registers / 2 CTAs, 320^3); the queue then holds u1..u3
#ifndef CST_R4MINB
#define CST_R4MINB (65536 / (CST_TBX * CST_TBY * CST_TBZ * 168) > 0 ? 65536 / (CST_TBX * CST_TBY * CST_TBZ * 168) : 1)
#endif
#define CST_LB __launch_bounds__(CST_TBX * CST_TBY * CST_TBZ, CST_R4MINB)
#elif defined(CST_MINB)  // experiment hook (CST_NVRTC_DEFINES="-DCST_MINB=n")
#define CST_LB __launch_bounds__(CST_TBX * CST_TBY * CST_TBZ, CST_MINB)
#else
#define CST_LB __launch_bounds__(CST_TBX * CST_TBY * CST_TBZ)
#endif
// R12: every smem-staged row is read as 16-B pairs somewhere (x windows, walks), so its
// length T_x + 2 XR must be even (a 1 x 32 ld/st tile faulted with a misaligned address)
static_assert(STAGING == 1 || TX % 2 == 0, "R12: smem staging needs an even tile extent T_x");
extern "C" __global__ void CST_LB cst_kernel(const __grid_constant__ cst_kparams P) {
  extern __shared__ __align__(128) double cst_smem[];
  if constexpr (BT > 1) {
    kernel_tblock<0>(P, cst_smem);
  } else if constexpr (!STREAM) {
    kernel_tile3d(P, cst_smem);
  } else if constexpr (R4RET) {
    kernel_rhs4_ret<0>(P, cst_smem);
  } else if constexpr (QTM && KIND == 3) {
    kernel_hyp_tmem<0>(P, cst_smem);
  } else if constexpr (QTM) {
    kernel_star_tmem<0>(P, cst_smem);
  } else if constexpr ((KIND == 1 || KIND == 2) && TS == 1) {
    kernel_stream1(P, cst_smem);
  } else if constexpr (KIND == 3 && TS == 1) {
    kernel_hyp_stream1(P, cst_smem);
  } else {
    kernel_stream_generic(P, cst_smem);
  }
}
