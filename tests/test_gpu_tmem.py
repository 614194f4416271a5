"""GPU parity of the TMEM streamed-state path (field 21, qstore = 2).

The star's retimed sweep with its per-point ring of (value, partial output) pairs in
tensor memory instead of registers.  Same inputs as the oracle (cstgen, host), ragged grids
with a NaN-poisoned outer halo ring, several streaming chunks, every order 1..4, both
streaming axes, multi-step ping-pong; tolerance = north_star 1e-12 relative max-norm.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402
import gpu_helpers as H  # noqa: E402
from test_gpu_sweep import run_gpu  # noqa: E402

pytestmark = pytest.mark.gpu


def Q(**kw):
    d = dict(tb_x=32, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=8,
             uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=2, bm_y=2, bm_z=1,
             use_retiming=2, prefetch=2, bt=1, qstore=2)
    d.update(kw)
    return C.cst_setting.from_dict(d)


CASES = [
    ("bm2x2", Q()),
    ("bm4x4", Q(bm_x=4, bm_y=4, tb_x=16, tb_y=4)),
    ("bm2x4-8warps", Q(bm_y=4, tb_x=16, tb_y=8)),
    ("bm1x1-pf1", Q(bm_x=1, bm_y=1, prefetch=1)),
    ("bm4x2-pf4-sb16", Q(bm_x=4, tb_x=8, tb_y=8, prefetch=4, sb=16)),
    ("cm2", Q(tb_x=16, cm_x=2, bm_x=1)),
    ("const-mem", Q(use_constant=2)),
    ("sd-y", Q(tb_y=1, tb_z=4, sd=2, bm_y=1, bm_z=2)),
    ("sb1", Q(sb=1, prefetch=1)),
]


@pytest.mark.parametrize("r", [1, 2, 3, 4])
@pytest.mark.parametrize("name,setting", CASES, ids=[c[0] for c in CASES])
def test_star_tmem_ragged(name, setting, r):
    kind = 1
    L = H.layout((75, 37, 22), r + 1)           # extra halo ring poisoned with NaN
    c = H.coeffs(kind, r, "random", seed=r)
    ins = H.inputs(kind, L, seed=7 + r, poison_beyond=r)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    _, got = run_gpu(kind, r, c, L, ins, setting)
    H.assert_parity(L, got[0], want[0], f"{name} r={r}")
    H.assert_halo_untouched(L, got[0], np.full(L.numel, np.nan))


def test_star_tmem_multistep():
    kind, r = 1, 4
    L = H.layout((40, 33, 30), r)
    c = H.coeffs(kind, r)
    ins = H.inputs(kind, L, seed=11)
    _, want = H.oracle_outputs(kind, r, c, L, ins, nsteps=3)
    init = [b.copy() for b in ins]
    _, gout = run_gpu(kind, r, c, L, ins, Q(bm_x=4, bm_y=4, tb_x=8, tb_y=4), nsteps=3,
                        out_init=init)
    H.assert_parity(L, gout[0], want[0], "3 steps")


def test_star_tmem_polynomial_bit_exact():
    """Integer weights on a degree-<=2r polynomial field: every partial sum is an exact
    integer, so the TMEM path's summation order cannot change a bit."""
    kind, r = 1, 2
    L = H.layout((34, 20, 18), r)
    w = [-1.0, 16.0, -30.0, 16.0, -1.0]
    c = [3 * w[2]] + [w[0], w[1], w[3], w[4]] * 3
    z, y, x = np.meshgrid(np.arange(L.nz + 2 * r), np.arange(L.ny + 2 * r),
                          np.arange(L.pitch_x), indexing="ij")
    f = np.zeros(L.numel)
    v = L.view(f)
    v[...] = (x * x + 2 * y * z - 3 * z * z + x)[:, :, :v.shape[2]]
    ins = [f]
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    _, got = run_gpu(kind, r, c, L, ins, Q(bm_x=4, bm_y=4, tb_x=8, tb_y=4))
    gi, wi = H.interior(L, got[0]), H.interior(L, want[0])
    assert np.array_equal(gi, wi)


def test_tmem_space_rule_and_default_unchanged():
    g = C.make_grid(64, 64, 64, 4)
    h = C.cst_stencil_create(1, 4, [1.0] * 25, g)
    try:
        assert C.cst_setting_default(h).qstore == 1
        C.cst_setting_check(h, Q(bm_x=4, bm_y=4, tb_x=16))
        with pytest.raises(C.CstError):
            C.cst_setting_check(h, Q(staging=2))          # R15
    finally:
        C.cst_stencil_destroy(h)


HYP_CASES = [
    ("z-32x4", Q(tb_x=32, tb_y=4, bm_x=1, bm_y=1, sb=8)),
    ("z-16x8-pf3", Q(tb_x=16, tb_y=8, bm_x=1, bm_y=1, prefetch=3, sb=16)),
    ("y-16x1x8", Q(tb_x=16, tb_y=1, tb_z=8, sd=2, bm_x=1, bm_y=1, sb=8)),
    ("y-16x1x16-const", Q(tb_x=16, tb_y=1, tb_z=16, sd=2, bm_x=1, bm_y=1, sb=16,
                          use_constant=2, prefetch=3)),
    ("sb1-pf1", Q(tb_x=32, tb_y=4, bm_x=1, bm_y=1, sb=1, prefetch=1)),
    # two points stacked along b (BM_b = 2): union of the b-windows, per-point TMEM rings
    ("z-32x4-bmy2", Q(tb_x=32, tb_y=4, bm_x=1, bm_y=2, sb=8)),
    ("z-16x8-bmy2-pf3", Q(tb_x=16, tb_y=8, bm_x=1, bm_y=2, prefetch=3, sb=16, use_constant=2)),
    ("y-32x1x4-bmz2", Q(tb_x=32, tb_y=1, tb_z=4, sd=2, bm_x=1, bm_y=1, bm_z=2, sb=8)),
]


@pytest.mark.parametrize("name,setting", HYP_CASES, ids=[c[0] for c in HYP_CASES])
def test_hypterm_tmem_ragged(name, setting):
    """hypterm-like (8 inputs, 5 outputs, order 4) with the 45-double streamed state in a
    TMEM ring: every output within 1e-12 of the oracle, halos untouched."""
    kind, r = 3, 4
    L = H.layout((37, 29, 26), r + 1)
    c = H.coeffs(kind, r, "random", seed=3)
    ins = H.inputs(kind, L, seed=13, poison_beyond=r)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    _, got = run_gpu(kind, r, c, L, ins, setting)
    for o in range(5):
        H.assert_parity(L, got[o], want[o], f"{name} out{o}")
        H.assert_halo_untouched(L, got[o], np.full(L.numel, np.nan))


def test_hypterm_tmem_matches_register_path():
    """Same setting with the state in registers (qstore 1) and in TMEM (qstore 2): the two
    differ only in summation order."""
    kind, r = 3, 4
    L = H.layout((48, 40, 36), r)
    c = H.coeffs(kind, r)
    ins = H.inputs(kind, L, seed=21)
    d = dict(tb_x=16, tb_y=1, tb_z=8, sd=2, bm_x=1, bm_y=1, sb=16, prefetch=3)
    _, a = run_gpu(kind, r, c, L, ins, Q(qstore=1, **d))
    _, b = run_gpu(kind, r, c, L, ins, Q(qstore=2, **d))
    for o in range(5):
        H.assert_parity(L, b[o], a[o], f"out{o}")
