"""Pins of the tuner / space oracle (oracle/tuner.py, oracle/space.py) — CPU only.

Worked examples discriminate the readings of the garbled listings (Algorithm 1: text vs
listing, P:162 vs P:170-230; Algorithm 2); closed forms and library routines
(numpy corrcoef, lstsq) pin the statistics; the Fig. 7 example pins re-indexing;
the literal Table I counts (">100 million") were computed independently during the
survey.
"""
import json
import math
import os

import numpy as np
import pytest

from oracle import space as S
from oracle import tuner as T

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_cv_eq1_closed_form():
    assert abs(T.cv([1, 2, 3, 4]) - math.sqrt(1.25) / 2.5) < 1e-15
    assert abs(T.cv([1, 2, 3, 4]) - 0.4472135955) < 1e-10
    assert T.cv([3, 3, 3]) == 0.0 and T.cv([0, 0]) == 0.0


def test_pcc_matches_numpy():
    rng = np.random.default_rng(0)
    for _ in range(20):
        x, y = rng.normal(size=50), rng.normal(size=50)
        y = y + rng.uniform(-2, 2) * x
        assert abs(T.pcc(x, y) - np.corrcoef(x, y)[0, 1]) < 1e-14
    assert T.pcc([1, 1, 1], [1, 2, 3]) == 0.0


def test_algorithm1_worked_example_text_reading():
    A, B, C, D = range(4)
    dq = [(A, B), (C, D), (A, C), (B, D), (B, C), (A, D)]      # ascending CV
    assert T.group_parameters(dq) == [[A, B], [D, C]]
    # (the listing reading would give [[A, D], [B], [C]]: SURVEY §8(c) Q6)


def test_algorithm1_groups_every_parameter():
    rng = np.random.default_rng(3)
    n = 7
    pairs = [((a, b), float(rng.uniform())) for a in range(n) for b in range(n) if a != b]
    groups = T.group_parameters(T.ascending_deque(pairs))
    flat = sorted(p for g in groups for p in g)
    assert flat == list(range(n))


def test_algorithm2_worked_example():
    m1, m2, m3, m4, m5, m6 = range(6)
    by_abs = [((m4, m5), .05), ((m2, m3), .1), ((m1, m3), -.2), ((m2, m4), .3), ((m1, m4), .4),
              ((m5, m6), .5), ((m3, m4), -.9), ((m1, m2), .95)]
    dq = T.ascending_deque(by_abs, key=abs)
    assert T.combine_metrics(dq, 2) == [[m1, m2], [m3, m4, m5]]
    assert T.combine_metrics(dq, 3) == [[m1, m2], [m3, m4], [m5, m6]]


def test_select_metric_highest_abs_pcc_with_time():
    rng = np.random.default_rng(1)
    t = rng.normal(size=40)
    M = np.stack([rng.normal(size=40), -3 * t + 0.01 * rng.normal(size=40), t + rng.normal(size=40)], 1)
    assert T.select_metrics([[0, 1, 2]], M, t) == [1]


def test_pair_cv_dataset_reading():
    # 2 fields a, b (both pow2).  rows: best row with a=1 has b=4, best with a=2 has b=1.
    rows = [({"a": 1, "b": 4}, 0), ({"a": 1, "b": 2}, 1), ({"a": 2, "b": 1}, 2), ({"a": 2, "b": 8}, 3)]
    fit = [5.0, 1.0, 7.0, 7.0]           # tie at a=2 -> lower rank (row 2, b=1)
    T.POW2_FIELDS.update({"a", "b"})
    out = dict(T.pair_cvs(rows, fit, fields=("a", "b")))
    assert out[(0, 1)] == T.cv([2.0, 0.0])          # VS_ab = log2 (4, 1) = (2, 0)
    # VS_ba: b=1 -> a=2 ; b=2 -> a=1 ; b=4 -> a=1 ; b=8 -> a=2  (log2: 1,0,0,1)
    assert out[(1, 0)] == T.cv([1.0, 0.0, 0.0, 1.0])


def test_pmnf_recovers_generating_hypothesis():
    rng = np.random.default_rng(7)
    groups = [[0, 1], [2]]
    X = 2 ** rng.integers(0, 7, size=(128, 3))
    for (i, j) in [(1, 0), (2, 1), (1, 1)]:
        c = np.array([0.37, -1.25])
        y = T.pmnf_features(groups, X, i, j) @ c
        fits, best = T.pmnf_fit(groups, X, y)
        assert (fits[best][0], fits[best][1]) == (i, j)
        assert np.allclose(fits[best][2], c, rtol=1e-10, atol=0)
        assert fits[best][3] < 1e-12 * np.max(np.abs(y))


def test_pmnf_rse_formula():
    rng = np.random.default_rng(8)
    X = 2 ** rng.integers(0, 5, size=(40, 3))
    y = rng.normal(size=40)
    groups = [[0], [1, 2]]
    fits, _ = T.pmnf_fit(groups, X, y)
    for (i, j, coef, rse) in fits:
        A = T.pmnf_features(groups, X, i, j)
        rank = np.linalg.matrix_rank(A)
        ref_coef = np.linalg.pinv(A) @ y
        ssr = float(np.sum((y - A @ ref_coef) ** 2))
        assert abs(rse - math.sqrt(ssr / (40 - rank))) <= 1e-10 * max(1.0, rse)


def test_threshold_filter_fraction():
    rng = np.random.default_rng(2)
    preds = rng.normal(size=(1000, 2))
    t, th = T.threshold_filter(preds, [1, -1], 0.10)
    kept = [T.passes(p, [1, -1], th) for p in preds]
    assert np.mean(kept) >= 0.10
    if t > 0:                          # minimality: one index tighter falls below 10 %
        asc = [np.sort(preds[:, 0]), np.sort(preds[:, 1])]
        th2 = [asc[0][t - 1], asc[1][999 - (t - 1)]]
        assert np.mean([T.passes(p, [1, -1], th2) for p in preds]) < 0.10


def test_reindex_fig7_example():
    m = T.reindex([(0, 1), (4, 2), (3, 4)])
    assert [m[t] for t in [(0, 1), (4, 2), (3, 4)]] == [0, 2, 1]


def test_sampler_distinct_and_deterministic():
    a = T.sample_ranks(42, 10**9, 128)
    assert len(set(a)) == 128 and a == T.sample_ranks(42, 10**9, 128)
    assert all(0 <= x < 10**9 for x in a)
    assert T.sample_ranks(1, 50, 128) == list(range(50))
    with open(os.path.join(GOLD, "sampler.json")) as f:
        g = json.load(f)
    assert T.sample_ranks(g["seed"], g["count"], len(g["ranks"])) == g["ranks"]


# ----------------------------------------------------------------------------- space
def test_literal_table1_counts():
    """after the explicit constraints the space has > 100 million settings.
    Survey-computed literal counts ('Space enumeration' pin)."""
    want = {(4, 4, 4): 5.864e8, (64, 64, 64): 2.233e12, (320, 320, 320): 2.638e13,
            (512, 512, 512): 7.448e13}
    for M, w in want.items():
        n = S.literal_table1_count(M)
        assert abs(n - w) / w < 5e-4 and n > 1e8


def test_space_rules_spot_checks():
    base = dict(tb_x=32, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3,
                sb=64, uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=1, bm_y=1, bm_z=1,
                use_retiming=2, prefetch=2, bt=1, qstore=1)
    M = (512, 512, 512)
    assert S.check(1, 4, M, base) is None
    assert S.check(1, 4, M, dict(base, tb_x=64, tb_y=32)) == "R1"
    assert S.check(1, 4, M, dict(base, use_streaming=1)) == "R2"
    assert S.check(1, 4, M, dict(base, uf_z=128)) == "R3"
    assert S.check(1, 4, M, dict(base, tb_x=8, tb_y=2)) == "R4"
    assert S.check(1, 4, M, dict(base, tb_z=2, bm_z=64)) == "R5"
    assert S.check(1, 4, M, dict(base, uf_x=2)) == "R6"
    # R6 with the path's loop (round 2, tools/knob_audit.py): on the fast streaming path the
    # in-plane block is register-unrolled (no UF_x / UF_y loop) even when BM > 1; along z the
    # plane loop (<= SB) is unrolled for star/box with TMA, but not with ld/st staging, TMEM or
    # for the hypterm; the generic path (T_z > 1) unrolls the merged-point loop BM_z * CM_z
    assert S.check(1, 4, M, dict(base, bm_y=2, uf_y=2)) == "R6"
    assert S.check(1, 4, M, dict(base, uf_z=64)) is None
    assert S.check(1, 4, M, dict(base, uf_z=2, staging=2)) == "R6"
    assert S.check(1, 4, M, dict(base, uf_z=2, qstore=2)) == "R6"
    assert S.check(3, 4, M, dict(base, uf_z=2)) == "R6"
    assert S.check(1, 4, M, dict(base, tb_y=2, tb_z=2, uf_z=2)) == "R6"
    assert S.check(1, 4, M, dict(base, tb_y=2, tb_z=2, bm_z=2, uf_z=2)) is None
    assert S.check(1, 4, M, dict(base, use_streaming=1, sd=1, sb=1, prefetch=1, bm_y=2,
                                 uf_y=2)) is None
    # R9: no staging -> nothing to prefetch; R16: rhs4's retimed form only on its column
    # walk (T_SD = 1, TMA, bt 1, registers, CM 1, BM_b 1, BM_x <= 2)
    assert S.check(1, 4, M, dict(base, staging=1)) == "R9"
    assert S.check(1, 4, M, dict(base, staging=1, prefetch=1)) is None
    assert S.check(4, 2, M, dict(base, tb_x=16, tb_y=8)) is None
    assert S.check(4, 2, M, dict(base, tb_x=8, tb_y=8, bm_x=2)) is None
    assert S.check(4, 2, M, dict(base, tb_x=16, tb_y=8, use_retiming=1)) is None
    assert S.check(4, 2, M, dict(base, tb_x=16, tb_y=4, bm_y=2)) == "R16"
    assert S.check(4, 2, M, dict(base, tb_x=8, tb_y=8, bm_x=4)) == "R16"
    assert S.check(4, 2, M, dict(base, tb_x=16, tb_y=8, staging=2)) == "R16"
    assert S.check(4, 2, M, dict(base, tb_x=16, tb_y=4, tb_z=2)) == "R16"
    assert S.check(4, 2, M, dict(base, tb_x=8, tb_y=8, cm_x=2)) == "R16"
    assert S.check(4, 2, M, dict(base, tb_x=16, tb_y=8, uf_x=2)) == "R6"
    assert S.check(1, 4, M, dict(base, bm_y=8, cm_y=4)) == "R7"
    assert S.check(1, 4, M, dict(base, sd=1)) == "R8"
    assert S.check(1, 4, M, dict(base, use_streaming=1, sd=1, sb=1, prefetch=2)) == "R9"
    assert S.check(3, 4, M, dict(base, tb_x=128, tb_y=8, prefetch=4, use_retiming=1)) == "R10"
    assert S.check(3, 4, M, dict(base, bm_x=4)) == "R11"
    assert S.check(1, 4, M, dict(base, tb_x=128, tb_y=1)) is None
    assert S.check(1, 4, M, dict(base, tb_x=256, tb_y=1)) == "R12"
    assert S.check(1, 4, M, dict(base, tb_x=32, tb_y=1, bm_x=8)) == "R12"
    # ld/st staging: rows read as 16-B pairs need an even T_x (a 1 x 32 ld/st hypterm tile
    # faulted with a misaligned shared load on B200)
    assert S.check(3, 4, M, dict(base, tb_x=1, tb_y=32, staging=2, prefetch=1, sb=16)) == "R12"
    assert S.check(1, 4, M, dict(base, tb_x=1, tb_y=32, staging=2)) == "R12"
    assert S.check(1, 4, M, dict(base, tb_x=1, tb_y=32, staging=1, prefetch=1)) is None
    # temporal blocking (field 20): R14 structure, models by hand
    tb = dict(base, bm_x=2, bm_y=2, bt=2)
    assert S.check(2, 1, M, tb) is None
    assert S.check(3, 4, M, tb) == "R14"                       # hypterm: no fused path
    assert S.check(2, 1, M, dict(tb, staging=2)) == "R14"
    assert S.check(2, 1, M, dict(tb, use_retiming=1)) == "R14"
    assert S.check(2, 1, M, dict(tb, sd=2, sb=64)) == "R14"
    assert S.check(2, 1, M, dict(tb, uf_z=2)) == "R6"          # the fused kernel unrolls no plane loop
    assert S.check(2, 1, M, dict(tb, bm_x=4, tb_x=16)) == "R14"
    assert S.check(2, 1, M, dict(tb, cm_x=2, tb_x=16)) == "R14"
    # box r=1, tile 64x8, bt=2, 2 stages: input box (64+2*2*2)x(8+2*2) = 72x12 doubles
    # = 6912 B per ring slot; level 1 (64+4)x(8+2) = 680 doubles = 5440 B -> 5504 B slots
    assert S.smem_bytes(2, 1, tb) == 2 * 6912 + 2 * 5504
    # registers: level 1 has 34x5 = 170 blocks -> 2 per thread, level 2 128 -> 1; 3 blocks
    # x 4 points x 3 accumulators + a (2+2)x(2+4) window = 36 + 24 doubles
    assert S.est_regs(2, 1, tb) == 32 + 2 * (36 + 24)
    assert S.check(1, 4, M, dict(tb, bt=4)) == "R11"
    assert S.check(2, 1, M, dict(tb, tb_x=128, tb_y=1, bm_y=1)) == "R12"  # 256 + 8 > 256
    # TMEM streamed state (field 21): R15 structure + capacity, by hand
    q = dict(base, tb_x=32, tb_y=4, bm_x=4, bm_y=4, qstore=2)
    # 128 threads = 4 warps, one per lane quarter; 16 points x 4r = 16 columns -> 256
    assert S.tmem_columns(4, q) == 256 and S.check(1, 4, M, q) is None
    # registers: 2 doubles per point (in-plane part, centre) + ring (r + 1) + 2r
    assert S.est_regs(1, 4, q) == 32 + 2 * (32 + 5 + 8)
    assert S.check(1, 4, M, dict(base, bm_x=4, bm_y=4)) == "R11"  # same block in registers
    assert S.check(1, 4, M, dict(q, tb_y=8)) is None    # 8 warps: 2 per quarter -> 512
    assert S.tmem_columns(4, dict(q, tb_y=8)) == 512
    assert S.check(1, 4, M, dict(q, tb_y=16, bm_y=2)) is None   # 4 warps/quarter x 8 x 16
    assert S.check(1, 4, M, dict(q, tb_y=16, bm_y=4)) == "R15"  # 1024 columns
    # hypterm: one point per thread, 20r columns per point (5 products + 5 partial fluxes
    # per ring slot); 128 threads -> 80 columns, 1024 threads -> 8 warps/quarter -> 640
    hq = dict(base, qstore=2)
    assert S.tmem_columns(4, hq, 3) == 80 and S.check(3, 4, M, hq) is None
    assert S.est_regs(3, 4, hq) == 32 + 2 * (25 + 10 + 30)
    assert S.check(3, 4, M, dict(hq, bm_x=2, tb_x=16)) == "R15"   # blocked: not this path
    assert S.check(3, 4, M, dict(hq, tb_y=32)) == "R15"            # 640 columns
    # rhs4: the retimed column walk's s-window queue, 10 (2r + 1) = 50 columns per point
    assert S.tmem_columns(2, hq, 4) == 50 and S.check(4, 2, M, hq) is None
    assert S.check(4, 2, M, dict(hq, tb_x=16, bm_x=2)) is None     # 100 columns
    assert S.check(4, 2, M, dict(hq, tb_y=32, bm_x=2)) == "R15"    # 8 warps/quarter: 800
    assert S.check(4, 2, M, dict(hq, use_retiming=1)) == "R15"     # generic path: no TMEM
    assert S.check(1, 4, M, dict(q, staging=2)) == "R15"
    assert S.check(1, 4, M, dict(q, use_retiming=1)) == "R15"
    assert S.check(1, 4, M, dict(q, tb_z=2, tb_y=2)) == "R15"  # T_SD = 2
    assert S.check(1, 4, M, dict(q, sd=2, tb_y=1, tb_z=4, bm_y=1, bm_z=4)) is None


def test_space_enumeration_small_is_sorted_and_valid():
    for kind, r in [(1, 2), (2, 1), (3, 4)]:
        seq = [S.as_tuple(s) for s in S.enumerate_space(kind, r, (4, 4, 4))]
        assert seq == sorted(seq) and len(set(seq)) == len(seq) and len(seq) > 0
        for t in seq[::97]:
            assert S.check(kind, r, (4, 4, 4), dict(zip(S.FIELDS, t))) is None
