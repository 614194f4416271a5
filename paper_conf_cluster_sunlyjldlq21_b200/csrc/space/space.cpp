// space.cpp — the parameter space of Table I with the rules of DESIGN.md §3:
// explicit rules of P:149 (R1-R3), our semantics rules (R4-R9) and the
// implicit resource rules (R10-R12: "settings ... restricted by the usage of
// register and shared memory ... only non-spilled parameter settings are explored") and
// R14, the structural requirements of the temporally blocked path (field 20, bt), and
// R15, those of the TMEM streamed-state path (field 21, qstore).
//
// Canonical order: lexicographic over the 21 fields (Table I row order, bt, qstore), values
// ascending.  count / rank / unrank are exact (bit-exact with oracle/space.py).
#include <algorithm>
#include <atomic>
#include <cstring>

#include "../runtime/internal.h"

namespace cst {

const char* const kFieldNames[F_COUNT] = {
    "tb_x", "tb_y", "tb_z", "staging", "use_constant", "use_streaming", "sd", "sb",
    "uf_x", "uf_y", "uf_z", "cm_x", "cm_y", "cm_z", "bm_x", "bm_y", "bm_z",
    "use_retiming", "prefetch", "bt", "qstore"};

Tuple to_tuple(const cst_setting& s) {
  return Tuple{s.tb[0], s.tb[1], s.tb[2], s.staging, s.use_constant, s.use_streaming,
               s.sd, s.sb, s.uf[0], s.uf[1], s.uf[2], s.cm[0], s.cm[1], s.cm[2],
               s.bm[0], s.bm[1], s.bm[2], s.use_retiming, s.prefetch, s.bt, s.qstore};
}

cst_setting from_tuple(const Tuple& t) {
  cst_setting s;
  s.tb[0] = t[F_TBX]; s.tb[1] = t[F_TBY]; s.tb[2] = t[F_TBZ];
  s.staging = t[F_STAGING]; s.use_constant = t[F_CONST]; s.use_streaming = t[F_STREAM];
  s.sd = t[F_SD]; s.sb = t[F_SB];
  for (int d = 0; d < 3; ++d) {
    s.uf[d] = t[F_UFX + d];
    s.cm[d] = t[F_CMX + d];
    s.bm[d] = t[F_BMX + d];
  }
  s.use_retiming = t[F_RET]; s.prefetch = t[F_PF]; s.bt = t[F_BT]; s.qstore = t[F_QS];
  return s;
}

std::string setting_key(const cst_setting& s) {
  Tuple t = to_tuple(s);
  std::string k;
  for (int i = 0; i < F_COUNT; ++i) {
    if (i) k += ',';
    k += std::to_string(t[i]);
  }
  return k;
}

static const int64_t SMEM_LIMIT = 227 * 1024 - 1024;
static const int64_t REG_LIMIT = 255;

static int n_arrays(int kind) {
  return kind == CST_HYPTERM ? 8 : (kind == CST_RHS4 ? 5 : 1);
}
static int live_doubles(int kind, int r) {
  return kind == CST_STAR ? 2 * r + 2
                          : (kind == CST_BOX ? 12 : (kind == CST_HYPTERM ? 50 : 24));
}
static int retention(int kind, int r) { return kind == CST_BOX ? 2 * r : r; }

static void tiles(const Tuple& t, int64_t T[3]) {
  for (int d = 0; d < 3; ++d)
    T[d] = (int64_t)t[F_TBX + d] * t[F_BMX + d] * t[F_CMX + d];
}

static int64_t xr_of(int r) { return r + (r & 1); }
static int64_t rnd128(int64_t bytes) { return (bytes + 127) / 128 * 128; }

// temporally blocked CTA (bt > 1): level lv extents, level 0 = TMA input box, lv = bt the
// output tile (mirrors tb_wa / tb_wb in csrc/kernels/cst_kernels.cuh)
static void tb_extent(int r, const Tuple& t, int lv, int64_t* ex, int64_t* ey) {
  int64_t T[3];
  tiles(t, T);
  const int64_t k = t[F_BT] - lv;
  *ex = T[0] + 2 * xr_of(r) * k;
  *ey = T[1] + 2 * (int64_t)r * k;
}

static int64_t tb_blocks_per_thread(int r, const Tuple& t, int lv) {
  int64_t ex, ey;
  tb_extent(r, t, lv, &ex, &ey);
  const int64_t nthr = (int64_t)t[F_TBX] * t[F_TBY] * t[F_TBZ];
  return ((ex / t[F_BMX]) * (ey / t[F_BMY]) + nthr - 1) / nthr;
}

static int64_t tb_smem_bytes(int r, const Tuple& t) {
  int64_t e0x, e0y, e1x, e1y;
  tb_extent(r, t, 0, &e0x, &e0y);
  tb_extent(r, t, 1, &e1x, &e1y);
  return t[F_PF] * rnd128(e0x * e0y * 8) + (t[F_BT] - 1) * 2 * rnd128(e1x * e1y * 8);
}

// R15: the TMEM streamed-state path (qstore = 2): star or hypterm, streaming with
// T_SD = 1, TMA, retimed, bt = 1 (hypterm: one point along x, BM_b <= 2, CM = 1); ceil(threads / 128) warps
// share a TMEM lane quarter, each thread keeps 4r (star) or 20r (hypterm: 5 products + 5
// partial fluxes per ring slot) columns per point, 512 columns per SM (mirrors TM_* in
// csrc/kernels/cst_kernels.cuh)
static int64_t tmem_cols_kind(int kind, int r, const Tuple& t) {
  int64_t ppt = 1;
  for (int d = 0; d < 3; ++d) ppt *= (int64_t)t[F_BMX + d] * t[F_CMX + d];
  const int64_t nthr = (int64_t)t[F_TBX] * t[F_TBY] * t[F_TBZ];
  // rhs4 retimed: the s-window queue, 5 arrays x (2r + 1) planes x 2 columns per point
  const int64_t per = kind == CST_HYPTERM ? 20 * r : (kind == CST_RHS4 ? 10 * (2 * r + 1) : 4 * r);
  return (nthr / 32 + 3) / 4 * ppt * per;
}

int tmem_cols_alloc(int kind, int r, const Tuple& t) {
  const int64_t used = tmem_cols_kind(kind, r, t);
  int c = 32;
  while (c < used && c < 512) c *= 2;
  return c;
}

bool r4ret_path(int kind, const Tuple& t);

static bool qs_path_ok(int kind, int r, const Tuple& t) {
  if (kind == CST_RHS4) return r4ret_path(kind, t) && tmem_cols_kind(kind, r, t) <= 512;
  if ((kind != CST_STAR && kind != CST_HYPTERM) || t[F_STREAM] != 2 || t[F_STAGING] != 3 ||
      t[F_RET] != 2 || t[F_BT] != 1)
    return false;
  const int sd = t[F_SD] - 1;
  if ((int64_t)t[F_TBX + sd] * t[F_BMX + sd] * t[F_CMX + sd] != 1) return false;
  if (kind == CST_HYPTERM) {  // one point along a (x), up to two stacked along b
    const int b = sd == 2 ? 1 : 2;
    for (int d = 0; d < 3; ++d)
      if (t[F_CMX + d] != 1 || (d != b && t[F_BMX + d] != 1) || t[F_BMX + d] > 2) return false;
  }
  return tmem_cols_kind(kind, r, t) <= 512;
}

// R16: rhs4's retimed kernel (kernel_rhs4_ret in csrc/kernels/cst_kernels.cuh): streaming
// with T_SD = 1, TMA, bt = 1, no cyclic merging, one point along b, BM_a <= 2; the s-window
// queue in registers / shared memory (qstore 1) or tensor memory (qstore 2, R15 columns)
bool r4ret_path(int kind, const Tuple& t) {
  if (kind != CST_RHS4 || t[F_RET] != 2) return false;
  if (t[F_STREAM] != 2 || t[F_STAGING] != 3 || t[F_BT] != 1) return false;
  const int sd = t[F_SD] - 1;
  const int b = sd == 2 ? 1 : 2;
  for (int d = 0; d < 3; ++d)
    if (t[F_CMX + d] != 1) return false;
  return t[F_TBX + sd] == 1 && t[F_BMX + sd] == 1 && t[F_BMX + b] == 1 && t[F_BMX] <= 2;
}

static bool tb_path_ok(int kind, const Tuple& t) {
  return (kind == CST_STAR || kind == CST_BOX) && t[F_STREAM] == 2 && t[F_SD] == 3 &&
         t[F_STAGING] == 3 && t[F_RET] == 2 && t[F_TBZ] == 1 && t[F_BMZ] == 1 &&
         t[F_CMX] == 1 && t[F_CMY] == 1 && t[F_CMZ] == 1 && t[F_BMX] <= 2 && t[F_BMY] <= 2 &&
         t[F_UFX] == 1 && t[F_UFY] == 1 && t[F_UFZ] == 1;
}

// (P, NP): in-plane (or 3-D box) elements and ring planes of the modelled staging
static void plane_geometry(int kind, int r, const Tuple& t, int64_t* P, int64_t* NP) {
  int64_t T[3];
  tiles(t, T);
  if (t[F_STREAM] == 1) {
    *P = (T[0] + 2 * r) * (T[1] + 2 * r) * (T[2] + 2 * r);
    *NP = 1;
    return;
  }
  const int sd = t[F_SD] - 1;
  int a = -1, b = -1;
  for (int d = 0; d < 3; ++d)
    if (d != sd) (a < 0 ? a : b) = d;
  *P = (T[a] + 2 * r) * (T[b] + 2 * r);
  const int64_t D = t[F_PF];
  if (T[sd] == 1 && r4ret_path(kind, t))
    *NP = D + 2 * r;  // + the 6 product planes (model_smem_bytes)
  else if (T[sd] == 1)
    *NP = D + (t[F_RET] == 2 ? 0 : retention(kind, r));
  else
    *NP = D * T[sd] + 2 * r;
}

// x-product planes of the TMEM hypterm kernel (hyp_prod_a in csrc/kernels/cst_kernels.cuh):
// two buffers of 5 products over the tile and its x-halo
static int64_t hyp_xprod_bytes(int kind, int r, const Tuple& t) {
  if (kind != CST_HYPTERM || t[F_QS] != 2 || t[F_STREAM] != 2) return 0;
  int64_t T[3];
  tiles(t, T);
  const int b = (t[F_SD] - 1) == 2 ? 1 : 2;
  return 2 * 5 * rnd128((T[0] + 2 * xr_of(r)) * T[b] * 8);
}

int64_t model_smem_bytes(int kind, int r, const Tuple& t) {
  if (t[F_STAGING] == 1) return 0;
  if (t[F_BT] > 1) return tb_smem_bytes(r, t);
  int64_t P, NP;
  plane_geometry(kind, r, t, &P, &NP);
  const int64_t plane = (P * 8 + 127) / 128 * 128;
  return (n_arrays(kind) * NP + (r4ret_path(kind, t) ? 6 : 0)) * plane +
         hyp_xprod_bytes(kind, r, t);
}

// Per-array halos of the hypterm TMA fast path (HTRIM in csrc/kernels/cst_kernels.cuh):
// array a's staged in-plane box is (T_a + 2 XR h_a) x (T_b + 2 r h_b) with h_a = 0 for q_b
// and q_s, h_b = 0 for q_a and q_s (inputs: cons1..4 = 0..3, q1..q3 = 4..6, q4 = 7).
bool hyp_trimmed(int kind, const Tuple& t) {
  if (kind != CST_HYPTERM || t[F_STAGING] != 3 || t[F_STREAM] != 2 || t[F_BT] != 1) return false;
  const int sd = t[F_SD] - 1;
  return (int64_t)t[F_TBX + sd] * t[F_BMX + sd] * t[F_CMX + sd] == 1;
}

void stream_array_box(int kind, int r, const Tuple& t, int a, int64_t* wa, int64_t* wb) {
  int64_t T[3];
  tiles(t, T);
  const int sd = t[F_SD] - 1;
  const int b = sd == 2 ? 1 : 2;
  const int q_a = 4, q_b = 4 + b;
  const bool trim = hyp_trimmed(kind, t);
  const bool ha = !trim || a < 4 || a == 7 || a == q_a;
  const bool hb = !trim || a < 4 || a == 7 || a == q_b;
  *wa = T[0] + (ha ? 2 * xr_of(r) : 0);
  *wb = T[b] + (hb ? 2 * (int64_t)r : 0);
}

int64_t kernel_smem_bytes(int kind, int r, const Tuple& t) {
  // mirrors csrc/kernels/cst_kernels.cuh: x halo XR = r rounded up to even
  if (t[F_STAGING] == 1) return 0;
  if (t[F_BT] > 1) return tb_smem_bytes(r, t) + 2 * (int64_t)t[F_PF] * 8;  // + mbarriers
  const int64_t XR = r + (r & 1);
  int64_t T[3];
  tiles(t, T);
  int64_t plane_elems, NP;
  if (t[F_STREAM] == 1) {
    plane_elems = (T[0] + 2 * XR) * (T[1] + 2 * r) * (T[2] + 2 * r);
    NP = 1;
  } else {
    const int sd = t[F_SD] - 1;
    const int b = sd == 2 ? 1 : 2;
    plane_elems = (T[0] + 2 * XR) * (T[b] + 2 * r);
    const int64_t D = t[F_PF];
    if (r4ret_path(kind, t))              // rhs4 retimed: planes c-2 .. c+2 + prefetch
      NP = D + 2 * r;
    else if (T[sd] == 1 && kind != CST_RHS4)  // fast streaming paths
      NP = D + (t[F_RET] == 2 ? 0 : retention(kind, r));
    else                                 // generic ring
      NP = D * T[sd] + 2 * r;
  }
  const int64_t plane = (plane_elems * 8 + 127) / 128 * 128;
  const int64_t bars = t[F_STAGING] == 3 ? 2 * NP * 8 : 0;  // full (+ optional empty) mbarriers
  if (t[F_STREAM] == 2 && r4ret_path(kind, t))  // + 2 buffers x 3 product planes
    return (n_arrays(kind) * NP + 6) * plane + bars;
  if (t[F_STREAM] == 2 && hyp_trimmed(kind, t)) {
    int64_t slot = 0;
    for (int a = 0; a < n_arrays(kind); ++a) {
      int64_t wa, wb;
      stream_array_box(kind, r, t, a, &wa, &wb);
      slot += rnd128(wa * wb * 8);
    }
    return NP * slot + hyp_xprod_bytes(kind, r, t) + bars;
  }
  return n_arrays(kind) * NP * plane + bars;
}

int64_t model_regs(int kind, int r, const Tuple& t) {
  if (r4ret_path(kind, t)) {
    // per point: s-window queue (5 arrays x 5 planes; 3 arrays when BM_a = 2, mu / lambda
    // then from the ring), 5 x 3 pending outputs, ~20 operands in flight
    return 32 + 2 * t[F_BMX] * (t[F_BMX] == 1 ? 60 : 50);
  }
  if (t[F_QS] == 2 && kind == CST_HYPTERM) {  // products, partial fluxes, ring, row values
    int64_t ppt = 1;
    for (int d = 0; d < 3; ++d) ppt *= (int64_t)t[F_BMX + d] * t[F_CMX + d];
    return 32 + 2 * (5 * (r + 1) + 10 * ppt + 30);
  }
  if (t[F_QS] == 2) {
    // TMEM path: in-plane part + centre per point, one point's ring (r + 1 doubles) and
    // the column windows of the block in flight
    int64_t ppt = 1;
    for (int d = 0; d < 3; ++d) ppt *= (int64_t)t[F_BMX + d] * t[F_CMX + d];
    return 32 + 2 * (2 * ppt + (r + 1) + 2 * r);
  }
  if (t[F_BT] > 1) {
    int64_t pts = 0;
    for (int lv = 1; lv <= t[F_BT]; ++lv) pts += tb_blocks_per_thread(r, t, lv);
    pts *= (int64_t)t[F_BMX] * t[F_BMY];
    const int64_t win = (t[F_BMY] + 2 * (int64_t)r) * (t[F_BMX] + 2 * xr_of(r));
    return 32 + 2 * ((2 * r + 1) * pts + win);
  }
  int64_t ppt = 1;
  for (int d = 0; d < 3; ++d) ppt *= (int64_t)t[F_BMX + d] * t[F_CMX + d];
  const int64_t nthr = (int64_t)t[F_TBX] * t[F_TBY] * t[F_TBZ];
  int64_t pf = 0;
  if (t[F_STAGING] == 2 && t[F_PF] > 1) {
    int64_t P, NP;
    plane_geometry(kind, r, t, &P, &NP);
    int64_t T[3];
    tiles(t, T);
    const int64_t per_step = t[F_STREAM] == 2 ? T[t[F_SD] - 1] : 1;
    pf = (t[F_PF] - 1) * ((n_arrays(kind) * P * per_step + nthr - 1) / nthr);
  }
  return 32 + 2 * ppt * live_doubles(kind, r) + 2 * pf;
}

static bool tma_ok(int r, const Tuple& t) {
  int64_t T[3];
  tiles(t, T);
  if (T[0] % 2) return false;
  if (t[F_BT] > 1) {
    int64_t ex, ey;
    tb_extent(r, t, 0, &ex, &ey);
    return ex <= 256 && ey <= 256;
  }
  for (int d = 0; d < 3; ++d) {
    const bool streamed = t[F_STREAM] == 2 && d == t[F_SD] - 1;
    const int64_t e = streamed ? T[d] : T[d] + 2 * r;
    if (e > 256) return false;
  }
  return true;
}

// R6: trip count of the per-thread loop the kernel path unrolls along dim d (loop
// unrolling); 1 where the path has no such loop, so UF_d stays at its canonical 1
// and no two settings generate the same code (tools/knob_audit.py).  Streaming off and
// generic streaming (T_SD > 1, rhs4): the merged-point loop BM_d*CM_d.  Fast streaming
// paths (star/box/hypterm, T_SD = 1): no in-plane loop; along SD the plane loop (SB), which
// is unrolled for star/box with TMA or no staging in the register-state, unfused kernel.
int64_t uf_trip(int kind, const Tuple& t, int d) {
  const int64_t bmcm = (int64_t)t[F_BMX + d] * t[F_CMX + d];
  if (t[F_STREAM] != 2) return bmcm;
  const int sd = t[F_SD] - 1;
  if (r4ret_path(kind, t)) return 1;  // rhs4 retimed: the pair is lockstep, the plane loop rolled
  const bool fast = (kind == CST_STAR || kind == CST_BOX || kind == CST_HYPTERM) &&
                    (int64_t)t[F_TBX + sd] * t[F_BMX + sd] * t[F_CMX + sd] == 1;
  if (!fast) return bmcm;
  if (d != sd) return 1;
  if ((kind == CST_STAR || kind == CST_BOX) && t[F_QS] == 1 && t[F_BT] == 1 &&
      t[F_STAGING] != 2)
    return t[F_SB];
  return 1;
}

static bool is_p2(int64_t v) { return v >= 1 && (v & (v - 1)) == 0; }

const char* check_rules(const StencilInfo& st, const Tuple& t) {
  // ranges (Table I)
  const int64_t* M = st.M;
  if (!is_p2(t[F_TBX]) || t[F_TBX] > 1024 || !is_p2(t[F_TBY]) || t[F_TBY] > 1024 ||
      !is_p2(t[F_TBZ]) || t[F_TBZ] > 64)
    return "range: TB";
  if (t[F_STAGING] < 1 || t[F_STAGING] > 3) return "range: staging";
  if (t[F_CONST] < 1 || t[F_CONST] > 2) return "range: use_constant";
  if (t[F_STREAM] < 1 || t[F_STREAM] > 2) return "range: use_streaming";
  if (t[F_SD] < 1 || t[F_SD] > 3) return "range: sd";
  if (!is_p2(t[F_SB]) || t[F_SB] > M[t[F_SD] - 1]) return "range: sb";
  for (int d = 0; d < 3; ++d) {
    if (!is_p2(t[F_UFX + d]) || t[F_UFX + d] > M[d]) return "range: uf";
    if (!is_p2(t[F_CMX + d]) || t[F_CMX + d] > M[d]) return "range: cm";
    if (!is_p2(t[F_BMX + d]) || t[F_BMX + d] > M[d]) return "range: bm";
  }
  if (t[F_RET] < 1 || t[F_RET] > 2) return "range: use_retiming";
  if (t[F_PF] < 1 || t[F_PF] > 4) return "range: prefetch";
  if (t[F_BT] != 1 && t[F_BT] != 2 && t[F_BT] != 4) return "range: bt";
  if (t[F_QS] < 1 || t[F_QS] > 2) return "range: qstore";

  const int64_t tb = (int64_t)t[F_TBX] * t[F_TBY] * t[F_TBZ];
  if (tb > 1024) return "R1";
  const bool stream = t[F_STREAM] == 2;
  if (!stream && (t[F_SD] != 1 || t[F_SB] != 1)) return "R2";
  if (stream && t[F_SD] == 1) return "R8";
  if (tb < 32) return "R4";
  int64_t T[3];
  tiles(t, T);
  const int sd = t[F_SD] - 1;
  for (int d = 0; d < 3; ++d) {
    const int64_t E = (stream && d == sd) ? t[F_SB] : M[d];
    if (T[d] > E) return "R5";
  }
  if (stream && t[F_UFX + sd] > t[F_SB]) return "R3";
  for (int d = 0; d < 3; ++d)
    if (t[F_UFX + d] > uf_trip(st.kind, t, d)) return "R6";
  int64_t ppt = 1;
  for (int d = 0; d < 3; ++d) ppt *= (int64_t)t[F_BMX + d] * t[F_CMX + d];
  if (ppt > 16) return "R7";
  if (t[F_PF] > 1 && (!stream || t[F_STAGING] == 1)) return "R9";
  if (t[F_BT] > 1 && !tb_path_ok(st.kind, t)) return "R14";
  if (t[F_QS] == 2 && !qs_path_ok(st.kind, st.r, t)) return "R15";
  if (st.kind == CST_RHS4 && t[F_RET] == 2 && !r4ret_path(st.kind, t)) return "R16";
  if (model_smem_bytes(st.kind, st.r, t) > SMEM_LIMIT) return "R10";
  if (model_regs(st.kind, st.r, t) > REG_LIMIT) return "R11";
  if (t[F_STAGING] == 3 && !tma_ok(st.r, t)) return "R12";
  // ld/st staging reads its rows as 16-B pairs too: the smem row (T_x + 2 XR) must be even
  if (t[F_STAGING] == 2 && T[0] % 2) return "R12";
  return nullptr;
}

// ------------------------------------------------------------------ enumerator
static std::vector<int32_t> p2_upto(int64_t hi) {
  std::vector<int32_t> v;
  for (int64_t x = 1; x <= hi; x *= 2) v.push_back((int32_t)x);
  return v;
}

static int32_t count_le(const std::vector<int32_t>& v, int64_t bound) {
  int32_t n = 0;
  for (int32_t x : v)
    if (x <= bound) ++n;
  return n;
}

void Space::cores_for(const int32_t* pre, std::vector<Core>* cores) const {
  cores->clear();
  Tuple t{};
  for (int i = 0; i < 8; ++i) t[i] = pre[i];
  t[F_UFX] = t[F_UFY] = t[F_UFZ] = 1;
  const bool stream = pre[F_STREAM] == 2;
  const int sd = pre[F_SD] - 1;
  for (int32_t cmx : p2_[0])
    for (int32_t cmy : p2_[1])
      for (int32_t cmz : p2_[2]) {
        if ((int64_t)cmx * cmy * cmz > 16) continue;
        for (int32_t bmx : p2_[0])
          for (int32_t bmy : p2_[1])
            for (int32_t bmz : p2_[2]) {
              if ((int64_t)cmx * cmy * cmz * bmx * bmy * bmz > 16) continue;
              const int32_t cm[3] = {cmx, cmy, cmz}, bm[3] = {bmx, bmy, bmz};
              bool cover = true;
              for (int d = 0; d < 3; ++d)
                if ((int64_t)pre[F_TBX + d] * cm[d] * bm[d] > st_.M[d]) cover = false;
              if (!cover) continue;
              for (int32_t ret = 1; ret <= 2; ++ret)
                for (int32_t pf = 1; pf <= 4; ++pf)
                  for (int32_t bt = 1; bt <= 4; bt *= 2)
                  for (int32_t qs = 1; qs <= 2; ++qs) {
                  for (int d = 0; d < 3; ++d) {
                    t[F_CMX + d] = cm[d];
                    t[F_BMX + d] = bm[d];
                  }
                  t[F_RET] = ret;
                  t[F_PF] = pf;
                  t[F_BT] = bt;
                  t[F_QS] = qs;
                  // UF is not part of the core: R14 needs UF = 1, which the UF counts
                  // below encode (a bt > 1 core admits only the first UF value per dim)
                  if (check_rules(st_, t) != nullptr) continue;
                  Core c;
                  for (int d = 0; d < 3; ++d) {
                    c.cm[d] = cm[d];
                    c.bm[d] = bm[d];
                    int64_t trip = uf_trip(st_.kind, t, d);
                    if (stream && d == sd) trip = std::min<int64_t>(trip, pre[F_SB]);  // R3
                    c.nuf[d] = bt > 1 ? 1 : count_le(p2_[d], trip);
                  }
                  c.ret = ret;
                  c.pf = pf;
                  c.bt = bt;
                  c.qs = qs;
                  cores->push_back(c);
                }
            }
      }
  // canonical core order: CMx, CMy, CMz, BMx, BMy, BMz, ret, pf, bt, qs
  std::stable_sort(cores->begin(), cores->end(), [](const Core& a, const Core& b) {
    const int32_t ka[10] = {a.cm[0], a.cm[1], a.cm[2], a.bm[0], a.bm[1], a.bm[2], a.ret, a.pf, a.bt, a.qs};
    const int32_t kb[10] = {b.cm[0], b.cm[1], b.cm[2], b.bm[0], b.bm[1], b.bm[2], b.ret, b.pf, b.bt, b.qs};
    return std::lexicographical_compare(ka, ka + 10, kb, kb + 10);
  });
}

static std::atomic<uint64_t> g_space_ids{0};

Space::Space(const StencilInfo& st) : st_(st), id_(++g_space_ids) {
  for (int d = 0; d < 3; ++d) p2_[d] = p2_upto(st.M[d]);
  const std::vector<int32_t> tbxy = p2_upto(1024), tbz = p2_upto(64);
  std::vector<Core> cores;
  uint64_t cum = 0;
  for (int32_t tbx : tbxy) {
    if (tbx > st.M[0]) continue;
    for (int32_t tby : tbxy) {
      if (tby > st.M[1] || (int64_t)tbx * tby > 1024) continue;
      for (int32_t tbzv : tbz) {
        const int64_t tb = (int64_t)tbx * tby * tbzv;
        if (tbzv > st.M[2] || tb > 1024 || tb < 32) continue;
        for (int32_t stg = 1; stg <= 3; ++stg)
          for (int32_t uc = 1; uc <= 2; ++uc)
            for (int32_t strm = 1; strm <= 2; ++strm)
              for (int32_t sd = 1; sd <= 3; ++sd) {
                if (strm == 1 && sd != 1) continue;
                if (strm == 2 && sd == 1) continue;
                const std::vector<int32_t> sbs =
                    strm == 2 ? p2_upto(st.M[sd - 1]) : std::vector<int32_t>{1};
                for (int32_t sb : sbs) {
                  Prefix p;
                  const int32_t v[8] = {tbx, tby, tbzv, stg, uc, strm, sd, sb};
                  std::memcpy(p.v, v, sizeof v);
                  cores_for(p.v, &cores);
                  uint64_t n = 0;
                  for (const Core& c : cores) n += (uint64_t)c.nuf[0] * c.nuf[1] * c.nuf[2];
                  if (n == 0) continue;
                  p.start = cum;
                  p.count = n;
                  cum += n;
                  prefixes_.push_back(p);
                }
              }
      }
    }
  }
  total_ = cum;
}

bool Space::at(uint64_t rank, Tuple* out) const {
  if (rank >= total_) return false;
  // prefix by binary search on start
  size_t lo = 0, hi = prefixes_.size();
  while (hi - lo > 1) {
    const size_t mid = (lo + hi) / 2;
    if (prefixes_[mid].start <= rank) lo = mid;
    else hi = mid;
  }
  const Prefix& P = prefixes_[lo];
  uint64_t q = rank - P.start;
  // the cores of the last prefix unranked on this thread are reused (sorted rank batches,
  // e.g. the tuner's quantile sample, mostly stay within one prefix)
  thread_local uint64_t c_space = 0;
  thread_local size_t c_prefix = (size_t)-1;
  thread_local std::vector<Core> cores;
  if (c_space != id_ || c_prefix != lo) {
    cores_for(P.v, &cores);
    c_space = id_;
    c_prefix = lo;
  }
  Tuple t{};
  for (int i = 0; i < 8; ++i) t[i] = P.v[i];
  // UF_x, UF_y, UF_z in turn: candidate value index u_d (0-based) allowed iff u_d < nuf[d]
  int32_t uidx[3] = {-1, -1, -1};
  for (int d = 0; d < 3; ++d) {
    bool found = false;
    for (int32_t u = 0; u < (int32_t)p2_[d].size(); ++u) {
      uint64_t cnt = 0;
      for (const Core& c : cores) {
        bool okc = true;
        for (int e = 0; e < d; ++e)
          if (uidx[e] >= c.nuf[e]) okc = false;
        if (!okc || u >= c.nuf[d]) continue;
        uint64_t m = 1;
        for (int e = d + 1; e < 3; ++e) m *= (uint64_t)c.nuf[e];
        cnt += m;
      }
      if (q < cnt) {
        uidx[d] = u;
        found = true;
        break;
      }
      q -= cnt;
    }
    if (!found) return false;
  }
  for (const Core& c : cores) {
    if (uidx[0] >= c.nuf[0] || uidx[1] >= c.nuf[1] || uidx[2] >= c.nuf[2]) continue;
    if (q == 0) {
      for (int d = 0; d < 3; ++d) {
        t[F_UFX + d] = p2_[d][uidx[d]];
        t[F_CMX + d] = c.cm[d];
        t[F_BMX + d] = c.bm[d];
      }
      t[F_RET] = c.ret;
      t[F_PF] = c.pf;
      t[F_BT] = c.bt;
      t[F_QS] = c.qs;
      *out = t;
      return true;
    }
    --q;
  }
  return false;
}

bool Space::rank(const Tuple& t, uint64_t* out) const {
  if (check_rules(st_, t) != nullptr) return false;
  // locate prefix (prefixes_ are in canonical order)
  const Prefix* P = nullptr;
  {
    size_t lo = 0, hi = prefixes_.size();
    while (lo < hi) {
      const size_t mid = (lo + hi) / 2;
      if (std::lexicographical_compare(prefixes_[mid].v, prefixes_[mid].v + 8, t.data(),
                                       t.data() + 8))
        lo = mid + 1;
      else
        hi = mid;
    }
    if (lo >= prefixes_.size() || !std::equal(t.data(), t.data() + 8, prefixes_[lo].v))
      return false;
    P = &prefixes_[lo];
  }
  std::vector<Core> cores;
  cores_for(P->v, &cores);
  int32_t uidx[3];
  for (int d = 0; d < 3; ++d) {
    uidx[d] = -1;
    for (int32_t u = 0; u < (int32_t)p2_[d].size(); ++u)
      if (p2_[d][u] == t[F_UFX + d]) uidx[d] = u;
    if (uidx[d] < 0) return false;
  }
  uint64_t q = 0;
  for (int d = 0; d < 3; ++d) {
    for (int32_t u = 0; u < uidx[d]; ++u) {
      for (const Core& c : cores) {
        bool okc = true;
        for (int e = 0; e < d; ++e)
          if (uidx[e] >= c.nuf[e]) okc = false;
        if (!okc || u >= c.nuf[d]) continue;
        uint64_t m = 1;
        for (int e = d + 1; e < 3; ++e) m *= (uint64_t)c.nuf[e];
        q += m;
      }
    }
  }
  for (const Core& c : cores) {
    if (uidx[0] >= c.nuf[0] || uidx[1] >= c.nuf[1] || uidx[2] >= c.nuf[2]) continue;
    bool same = c.ret == t[F_RET] && c.pf == t[F_PF] && c.bt == t[F_BT] && c.qs == t[F_QS];
    for (int d = 0; d < 3; ++d)
      same = same && c.cm[d] == t[F_CMX + d] && c.bm[d] == t[F_BMX + d];
    if (same) {
      *out = P->start + q;
      return true;
    }
    ++q;
  }
  return false;
}

}  // namespace cst
