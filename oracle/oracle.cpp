// oracle/oracle.cpp — plain, slow, obviously-correct CPU definition of the complex
// stencil sweep (SURVEY.md §8(c) O1–O5).  TEST INFRASTRUCTURE ONLY: only tests/,
// __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
// load liboracle.so.  It shares no code with the CUDA path (libcst); the only common
// module is the input generator cstgen/cst_gen.h, which holds no stencil arithmetic.
//
// Built with -O3 -fno-fast-math -ffp-contract=off (no FMA contraction), so every point
// is summed exactly in the order written below.  OpenMP parallelises only the outer z
// loop, which does not change any per-point result.
//
// Paper citations use P:n = /root/reference/PAPER.md line n.
//  * "order" = neighbour extent along each dimension (§I) = radius r.
//  * The stencil bodies are not printed in the paper (Table III, takes them
//    from [36]); the definitions below are DESIGN.md readings Q1/Q5, pinned by
//    tests/test_oracle_*.py (closed forms, polynomial exactness, scipy correlation,
//    impulse responses and the Table III FLOP count of hypterm).
#include <cmath>
#include <cstdint>
#include <cstring>
#include <vector>

#include "../cstgen/cst_gen.h"

namespace {

enum Kind { STAR = 1, BOX = 2, HYPTERM = 3, RHS4 = 4 };

struct Grid {
  int64_t nx, ny, nz, halo, lead_x, pitch_x, pitch_y;
  int64_t off(int64_t x, int64_t y, int64_t z) const {
    return ((z + halo) * pitch_y + (y + halo)) * pitch_x + lead_x + x;
  }
};

// ----------------------------------------------------------------------------------
// Point definitions, templated on the number type T so that a FLOP-counting type can
// run the very same code (oracle_hypterm_flops) — the Table III pin.
// `U(a, dx, dy, dz)` returns input array a at offset (dx, dy, dz) from the point.
// ----------------------------------------------------------------------------------

// O2 star (Table III shapes P:332-334):
//   out = c0*u + sum_{k=-r..-1,1..r} wx[k] u(p+k ex) + (same for y) + (same for z)
// coefficient layout [c0, wx[-r..-1], wx[1..r], wy[...], wz[...]] (6r+1 values);
// summation order: c0 term, then x (k ascending), then y, then z.
template <class T, class Acc>
void star_point(const Acc& U, int r, const double* c, T* out) {
  T s = T(c[0]) * U(0, 0, 0, 0);
  int idx = 1;
  for (int axis = 0; axis < 3; ++axis) {
    for (int k = -r; k <= r; ++k) {
      if (k == 0) continue;
      int dx = axis == 0 ? k : 0, dy = axis == 1 ? k : 0, dz = axis == 2 ? k : 0;
      s = s + T(c[idx]) * U(0, dx, dy, dz);
      ++idx;
    }
  }
  out[0] = s;
}

// O3 box (Table III "j3d27pt"): out = sum_{dz,dy,dx in [-r,r]} c[dz][dy][dx] u(p+d),
// coefficients z-major, summed dz, then dy, then dx ascending.
template <class T, class Acc>
void box_point(const Acc& U, int r, const double* c, T* out) {
  const int w = 2 * r + 1;
  T s = T(0.0);
  bool first = true;
  for (int dz = -r; dz <= r; ++dz)
    for (int dy = -r; dy <= r; ++dy)
      for (int dx = -r; dx <= r; ++dx) {
        T t = T(c[((dz + r) * w + (dy + r)) * w + (dx + r)]) * U(0, dx, dy, dz);
        s = first ? t : s + t;
        first = false;
      }
  out[0] = s;
}

// O4 hypterm-like (Table III "hypterm": order 4, 358 FLOPs, 13 I/O arrays, P:336;
// complex-stencil definition).  Inputs 0..7 = cons1..cons4, q1..q4; outputs
// flux0..flux4; coefficients [a1, a2, a3, a4, dxinv_x, dxinv_y, dxinv_z].
// Written exactly as the CNS "hypterm" loop body: per direction d the x pass assigns
// flux = -(...), the y and z passes subtract; products are formed pointwise at p±k e_d.
template <class T, class Acc>
void hypterm_point(const Acc& U, const double* c, T* flux) {
  enum { C1 = 0, C2, C3, C4, Q1, Q2, Q3, Q4 };
  const double a[4] = {c[0], c[1], c[2], c[3]};
  for (int d = 0; d < 3; ++d) {
    const T dxi = T(c[4 + d]);
    auto at = [&](int arr, int k) {
      return U(arr, d == 0 ? k : 0, d == 1 ? k : 0, d == 2 ? k : 0);
    };
    const int qd = Q1 + d;       // velocity component along d
    const int cd = C1 + d;       // momentum component along d (mass flux)
    T t[5];
    for (int f = 0; f < 5; ++f) {
      T sum = T(0.0);
      for (int k = 1; k <= 4; ++k) {
        T e;
        if (f == 0) {
          e = at(cd, k) - at(cd, -k);
        } else if (f <= 3) {
          const int cm = C1 + (f - 1);
          e = at(cm, k) * at(qd, k) - at(cm, -k) * at(qd, -k);
          if (f - 1 == d) e = e + (at(Q4, k) - at(Q4, -k));
        } else {
          e = at(C4, k) * at(qd, k) - at(C4, -k) * at(qd, -k) +
              (at(Q4, k) * at(qd, k) - at(Q4, -k) * at(qd, -k));
        }
        T term = T(a[k - 1]) * e;
        sum = (k == 1) ? term : sum + term;
      }
      t[f] = dxi * sum;
    }
    for (int f = 0; f < 5; ++f) flux[f] = (d == 0) ? -t[f] : flux[f] - t[f];
  }
}

// NEXT-1 rhs4center-like (Table III "rhs4center": order 2, 666 FLOPs, 8 I/O arrays, P:339;
// SW4 [1]; DESIGN.md §2 O7).  Inputs 0..4 = u1, u2, u3, mu, lambda; outputs r1..r3;
// coefficients [s_x, s_y, s_z] (direction scales).  The variable-coefficient elastic
// operator  r_i = sum_j d_j(mu (d_j u_i + d_i u_j)) + d_i(lambda div u)  with radius-2,
// 4th-order operators:
//   D_d[f]     = (f(-2) - 8 f(-1) + 8 f(+1) - f(+2)) / 12                (first derivative)
//   V_d[a](f)  = ( m1 (f(-2)-f(0)) + m2 (f(-1)-f(0)) + m3 (f(+1)-f(0)) + m4 (f(+2)-f(0)) ) / 6
//     m1 = a(-1) - 3/4 (a(0) + a(-2)),   m2 = a(-2) + a(+1) + 3 (a(0) + a(-1)),
//     m3 = a(-1) + a(+2) + 3 (a(+1) + a(0)),   m4 = a(+1) - 3/4 (a(0) + a(+2))
//   r_i = sum_d s_d^2 V_d[mu + delta_id (mu + lambda)](u_i)
//       + sum_{d != i} s_d s_i ( D_d[mu * D_i u_d] + D_i[lambda * D_d u_d] )
// summed in that order (d ascending); products are pointwise at the outer stencil's points.
template <class T, class Acc>
void rhs4_point(const Acc& U, const double* c, T* r) {
  enum { U1 = 0, U2, U3, MU, LA };
  auto sh = [](int d, int k, int* o) { o[0] = o[1] = o[2] = 0; o[d] = k; };
  for (int i = 0; i < 3; ++i) {
    T acc = T(0.0);
    for (int d = 0; d < 3; ++d) {
      // a(k) = mu(k) (+ mu(k) + lambda(k) on the diagonal d == i), along e_d
      auto a = [&](int k) {
        int o[3];
        sh(d, k, o);
        T m = U(MU, o[0], o[1], o[2]);
        if (d == i) return m + (m + U(LA, o[0], o[1], o[2]));
        return m;
      };
      auto f = [&](int k) {
        int o[3];
        sh(d, k, o);
        return U(U1 + i, o[0], o[1], o[2]);
      };
      const T am2 = a(-2), am1 = a(-1), a0 = a(0), ap1 = a(1), ap2 = a(2);
      const T m1 = am1 - T(0.75) * (a0 + am2);
      const T m2 = am2 + ap1 + T(3.0) * (a0 + am1);
      const T m3 = am1 + ap2 + T(3.0) * (ap1 + a0);
      const T m4 = ap1 - T(0.75) * (a0 + ap2);
      const T f0 = f(0);
      const T v = (m1 * (f(-2) - f0) + m2 * (f(-1) - f0) + m3 * (f(1) - f0) + m4 * (f(2) - f0)) *
                  T(1.0 / 6.0);
      const T term = (T(c[d]) * T(c[d])) * v;
      acc = (d == 0) ? term : acc + term;
    }
    for (int d = 0; d < 3; ++d) {
      if (d == i) continue;
      // D along `outer` of (coef array) * (D along `inner` of u_comp), products at the
      // outer stencil's points
      auto mixed = [&](int outer, int inner, int coef, int comp) {
        auto inner_d = [&](int ko) {
          auto at = [&](int ki) {
            int o[3] = {0, 0, 0};
            o[outer] += ko;
            o[inner] += ki;
            return U(comp, o[0], o[1], o[2]);
          };
          int o[3] = {0, 0, 0};
          o[outer] += ko;
          const T g = ((at(-2) - at(2)) + T(8.0) * (at(1) - at(-1))) * T(1.0 / 12.0);
          return U(coef, o[0], o[1], o[2]) * g;
        };
        return ((inner_d(-2) - inner_d(2)) + T(8.0) * (inner_d(1) - inner_d(-1))) *
               T(1.0 / 12.0);
      };
      const T sdi = T(c[d]) * T(c[i]);
      acc = acc + sdi * mixed(d, i, MU, U1 + d);   // d_d (mu d_i u_d)
      acc = acc + sdi * mixed(i, d, LA, U1 + d);   // d_i (lambda d_d u_d)
    }
    r[i] = acc;
  }
}

// FLOP-counting number type: counts + - * between counted values (negation is a sign
// flip, not a FLOP, matching Table III's convention as reconstructed in SURVEY §8(c)).
struct Flop {
  static inline int64_t count = 0;
  double v;
  Flop() : v(0) {}
  explicit Flop(double x) : v(x) {}
  friend Flop operator+(Flop a, Flop b) { ++count; return Flop(a.v + b.v); }
  friend Flop operator-(Flop a, Flop b) { ++count; return Flop(a.v - b.v); }
  friend Flop operator*(Flop a, Flop b) { ++count; return Flop(a.v * b.v); }
  Flop operator-() const { return Flop(-v); }
};

int n_inputs(int kind) { return kind == HYPTERM ? 8 : (kind == RHS4 ? 5 : 1); }
int n_outputs(int kind) { return kind == HYPTERM ? 5 : (kind == RHS4 ? 3 : 1); }

template <class Acc>
void point(int kind, int r, const double* c, const Acc& U, double* out) {
  if (kind == STAR) star_point<double>(U, r, c, out);
  else if (kind == BOX) box_point<double>(U, r, c, out);
  else if (kind == HYPTERM) hypterm_point<double>(U, c, out);
  else rhs4_point<double>(U, c, out);
}

bool valid_kind(int kind, int r) {
  if (kind == STAR) return r >= 1 && r <= 4;
  if (kind == BOX) return r == 1;
  if (kind == HYPTERM) return r == 4;
  if (kind == RHS4) return r == 2;
  return false;
}

}  // namespace

extern "C" {

// One sweep (or nsteps ping-pong sweeps) of the whole interior, O1: every interior
// point (x,y,z) in [0,nx)x[0,ny)x[0,nz) is updated from inputs on [-r, n+r); output
// halos are never written; with nsteps>1 the output of step t is the input of step t+1
// (needs n_in == n_out; halos of both buffers stay fixed = Dirichlet data).
// Returns 0 on success, nonzero on invalid arguments.
int oracle_sweep(int kind, int order, const double* coeffs, int64_t nx, int64_t ny,
                 int64_t nz, int64_t halo, int64_t lead_x, int64_t pitch_x, int64_t pitch_y,
                 double* const* in, double* const* out, int nsteps, int nthreads) {
  if (!valid_kind(kind, order) || halo < order || lead_x < halo ||
      pitch_x < lead_x + nx + halo || pitch_y < ny + 2 * halo || nsteps < 1)
    return 1;
  if (nsteps > 1 && n_inputs(kind) != n_outputs(kind)) return 2;
  const Grid G{nx, ny, nz, halo, lead_x, pitch_x, pitch_y};
  const int nin = n_inputs(kind), nout = n_outputs(kind);
  std::vector<double*> src(in, in + nin), dst(out, out + nout);
  for (int step = 0; step < nsteps; ++step) {
#pragma omp parallel for schedule(static) num_threads(nthreads > 0 ? nthreads : 1)
    for (int64_t z = 0; z < nz; ++z) {
      double res[5];  // up to 5 outputs
      for (int64_t y = 0; y < ny; ++y)
        for (int64_t x = 0; x < nx; ++x) {
          auto U = [&](int a, int dx, int dy, int dz) {
            return src[a][G.off(x + dx, y + dy, z + dz)];
          };
          point(kind, order, coeffs, U, res);
          for (int o = 0; o < nout; ++o) dst[o][G.off(x, y, z)] = res[o];
        }
    }
    if (nsteps > 1) std::swap(src[0], dst[0]);
  }
  return 0;
}

// Single interior point with inputs drawn straight from the generator (cstgen) at
// GLOBAL coordinates of an (nx, ny, nz_global) grid with halo `halo`; array ids are
// `array_id0 + a` for input a.  Lets tests check sampled outputs of full-size
// (512^3, 2048x1024^2) runs without materialising the inputs.  One sweep only.
int oracle_point_gen(int kind, int order, const double* coeffs, uint64_t seed,
                     int array_id0, int64_t nx, int64_t ny, int64_t halo, int64_t x,
                     int64_t y, int64_t z, double* out) {
  if (!valid_kind(kind, order)) return 1;
  uint64_t keys[8];  // up to 8 inputs
  for (int a = 0; a < n_inputs(kind); ++a) keys[a] = cstgen_key(seed, (uint64_t)(array_id0 + a));
  auto U = [&](int a, int dx, int dy, int dz) {
    return cstgen_value(keys[a], cstgen_index(nx, ny, halo, x + dx, y + dy, z + dz));
  };
  point(kind, order, coeffs, U, out);
  return 0;
}

// Number of floating-point operations the hypterm definition performs per point,
// counted by running hypterm_point on the counting type (Table III: 358).
int64_t oracle_hypterm_flops(void) {
  Flop::count = 0;
  const double c[7] = {1, 1, 1, 1, 1, 1, 1};
  auto U = [](int, int, int, int) { return Flop(1.0); };
  Flop f[5];
  hypterm_point<Flop>(U, c, f);
  return Flop::count;
}

int64_t oracle_rhs4_flops(void) {
  Flop::count = 0;
  const double c[3] = {1, 1, 1};
  auto U = [](int, int, int, int) { return Flop(1.0); };
  Flop f[3];
  rhs4_point<Flop>(U, c, f);
  return Flop::count;
}

int64_t oracle_star_flops(int r) {
  Flop::count = 0;
  std::vector<double> c(6 * r + 1, 1.0);
  auto U = [](int, int, int, int) { return Flop(1.0); };
  Flop f[1];
  star_point<Flop>(U, r, c.data(), f);
  return Flop::count;
}

int64_t oracle_box_flops(int r) {
  Flop::count = 0;
  std::vector<double> c((2 * r + 1) * (2 * r + 1) * (2 * r + 1), 1.0);
  auto U = [](int, int, int, int) { return Flop(1.0); };
  Flop f[1];
  box_point<Flop>(U, r, c.data(), f);
  return Flop::count;
}

}  // extern "C"
