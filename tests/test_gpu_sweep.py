"""GPU parity: libcst sweeps (through the C ABI) vs the CPU oracle on the same seeded inputs.

Inputs come from cstgen on the host (never from the CUDA path); the device generator is
separately shown bit-identical to cstgen.  Tolerance: north_star 1e-12 relative max-norm;
integer-weight polynomial pins must be bit-exact; halos/pads must be byte-identical.
"""
import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402
import cstgen  # noqa: E402
from oracle import stencil as ost  # noqa: E402
import gpu_helpers as H  # noqa: E402

pytestmark = pytest.mark.gpu


def _dev(a):
    return torch.from_numpy(a).cuda()


def run_gpu(kind, r, c, L, ins, setting, nsteps=1, out_init=None):
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    try:
        C.cst_setting_check(h, setting)
        dins = [_dev(b) for b in ins]
        if out_init is None:
            douts = [torch.full((L.numel,), float("nan"), dtype=torch.float64, device="cuda")
                     for _ in range(ost.N_OUT[kind])]
        else:
            douts = [_dev(b) for b in out_init]
        C.cst_sweep(h, setting, [t.data_ptr() for t in dins], [t.data_ptr() for t in douts],
                    nsteps, torch.cuda.current_stream().cuda_stream)
        C.cst_sync(h)
        return [t.cpu().numpy() for t in dins], [t.cpu().numpy() for t in douts]
    finally:
        C.cst_stencil_destroy(h)


def S(**kw):
    d = dict(tb_x=32, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=8,
             uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=1, bm_y=1, bm_z=1,
             use_retiming=2, prefetch=2)
    d.update(kw)
    return C.cst_setting.from_dict(d)


NOSTREAM = dict(use_streaming=1, sd=1, sb=1, prefetch=1)

# explicit coverage of every kernel path on a ragged grid
PATH_SETTINGS = [
    ("tma-retimed-pf2", S()),
    ("tma-retimed-pf1", S(prefetch=1)),
    ("tma-retimed-pf4", S(prefetch=4)),
    ("tma-gather-pf3", S(use_retiming=1, prefetch=3)),
    ("ldst-retimed-pf1", S(staging=2, prefetch=1)),
    ("ldst-retimed-pf3", S(staging=2, prefetch=3)),
    ("ldst-gather-pf2", S(staging=2, use_retiming=1)),
    ("none-retimed", S(staging=1, prefetch=1)),
    ("none-gather", S(staging=1, use_retiming=1, prefetch=1)),
    ("const-mem", S(use_constant=2)),
    ("sd-y", S(tb_y=1, tb_z=4, sd=2)),
    ("sd-y-ldst-gather", S(tb_y=1, tb_z=4, sd=2, staging=2, use_retiming=1)),
    ("merge-bm-cm", S(tb_x=16, cm_x=2, bm_y=2)),
    ("sb1", S(sb=1, prefetch=1)),
    ("generic-TS2-tma", S(tb_y=2, tb_z=2)),
    ("generic-TS2-ldst", S(tb_y=2, tb_z=2, staging=2)),
    ("generic-TS2-none", S(tb_y=2, tb_z=2, staging=1, prefetch=1)),
    ("generic-bmz2", S(bm_z=2, uf_z=1, sb=8)),
    ("tile3d-none", S(tb_x=16, tb_y=2, tb_z=2, staging=1, **NOSTREAM)),
    ("tile3d-ldst", S(tb_x=16, tb_y=2, tb_z=2, staging=2, **NOSTREAM)),
    ("tile3d-tma", S(tb_x=16, tb_y=2, tb_z=2, staging=3, **NOSTREAM)),
    ("tile3d-tma-merge", S(tb_x=16, tb_y=2, tb_z=1, staging=3, bm_z=2, cm_y=2, uf_z=2, **NOSTREAM)),
    ("tile3d-retimed", S(tb_x=16, tb_y=2, tb_z=2, staging=2, use_retiming=2, **NOSTREAM)),
    ("tb16-bm2x2", S(tb_x=16, tb_y=4, bm_x=2, bm_y=2)),
    ("tb16-bm2x4", S(tb_x=16, tb_y=2, bm_x=2, bm_y=4)),
]


@pytest.mark.parametrize("name,setting", PATH_SETTINGS, ids=[p[0] for p in PATH_SETTINGS])
def test_star_r2_paths_ragged(name, setting):
    kind, r = 1, 2
    L = H.layout((37, 29, 23), r + 1)           # extra halo ring poisoned with NaN
    c = H.coeffs(kind, r, "random", seed=1)
    ins = H.inputs(kind, L, seed=3, poison_beyond=r)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    _, got = run_gpu(kind, r, c, L, ins, setting)
    H.assert_parity(L, got[0], want[0], name)
    H.assert_halo_untouched(L, got[0], np.full(L.numel, np.nan))


@pytest.mark.parametrize("kind,r,n", [(1, 4, (64, 48, 40)), (1, 1, (33, 20, 17)),
                                      (1, 3, (40, 24, 30)), (2, 1, (50, 33, 27)),
                                      (3, 4, (40, 24, 20)), (4, 2, (36, 28, 20))])
def test_random_space_settings(kind, r, n):
    """Property-style: random valid settings drawn from the canonical space."""
    L = H.layout(n, r)
    c = H.coeffs(kind, r, "random", seed=kind + r)
    ins = H.inputs(kind, L, seed=5)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    cnt = C.cst_space_count(h)
    rng = random.Random(100 * kind + r)
    picks = [C.cst_setting_default(h)] + [C.cst_space_at(h, rng.randrange(cnt)) for _ in range(14)]
    C.cst_stencil_destroy(h)
    ran = 0
    for s in picks:
        try:
            _, got = run_gpu(kind, r, c, L, ins, s)
        except C.CstError as e:
            # implicit resource rule decided after code generation (R10 kernel smem, R13 spill)
            assert e.status == C.CST_E_CONSTRAINT, (s, e)
            continue
        ran += 1
        for o in range(ost.N_OUT[kind]):
            H.assert_parity(L, got[o], want[o], f"{s} out{o}")
    assert ran >= len(picks) // 2


@pytest.mark.parametrize("kind,r", [(1, 2), (1, 4), (2, 1), (3, 4), (4, 2)])
def test_config_coefficients_default_setting(kind, r):
    L = H.layout((64, 64, 64) if kind != 3 else (64, 32, 32), r)
    c = H.coeffs(kind, r)
    ins = H.inputs(kind, L, seed=kind)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    s = C.cst_setting_default(h)
    C.cst_stencil_destroy(h)
    _, got = run_gpu(kind, r, c, L, ins, s)
    for o in range(ost.N_OUT[kind]):
        H.assert_parity(L, got[o], want[o], f"out{o}")


RHS4_PAIRED = [("paired-tma", dict(tb_x=8, tb_y=8, bm_x=2)),
               ("paired-ldst", dict(tb_x=8, tb_y=8, bm_x=2, staging=2)),
               ("paired-bmy2", dict(tb_x=8, tb_y=4, bm_x=2, bm_y=2)),
               ("paired-sd-y", dict(tb_x=8, tb_y=1, tb_z=8, sd=2, bm_x=2)),
               ("scalar-bmx1", dict(tb_x=16, tb_y=8, bm_x=1))]


@pytest.mark.parametrize("name,kw", RHS4_PAIRED, ids=[p[0] for p in RHS4_PAIRED])
def test_rhs4_paired_points_ragged(name, kw):
    """rhs4 with BM_x = 2: the paired (two points per 16-B operand) evaluation, odd nx so
    the last pair of a row is half outside, poisoned far halo."""
    kind, r = 4, 2
    L = H.layout((37, 22, 19), r + 1)
    c = H.coeffs(kind, r, "random", seed=9)
    ins = H.inputs(kind, L, seed=13, poison_beyond=r)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    _, got = run_gpu(kind, r, c, L, ins, S(sb=8, uf_z=1, use_retiming=1, **kw))
    for o in range(ost.N_OUT[kind]):
        H.assert_parity(L, got[o], want[o], f"{name} out{o}")
        H.assert_halo_untouched(L, got[o], np.full(L.numel, np.nan))


RHS4_RETIMED = [("ret-pair-z", dict(tb_x=8, tb_y=8, bm_x=2)),
                ("ret-scalar-z", dict(tb_x=16, tb_y=8, bm_x=1)),
                ("ret-scalar-z-pf1", dict(tb_x=16, tb_y=8, bm_x=1, prefetch=1)),
                ("ret-pair-z-pf3-sb4", dict(tb_x=8, tb_y=4, bm_x=2, prefetch=3, sb=4)),
                ("ret-pair-y", dict(tb_x=16, tb_y=1, tb_z=8, sd=2, bm_x=2, prefetch=1)),
                ("ret-scalar-y-sb16", dict(tb_x=32, tb_y=1, tb_z=2, sd=2, bm_x=1, sb=16)),
                ("ret-pair-const", dict(tb_x=16, tb_y=2, bm_x=2, use_constant=2, prefetch=4)),
                # qstore 2: the s-window queue in tensor memory (R15)
                ("ret-pair-tmem", dict(tb_x=8, tb_y=16, bm_x=2, qstore=2, prefetch=1)),
                ("ret-pair-tmem-256thr", dict(tb_x=16, tb_y=16, bm_x=2, qstore=2, prefetch=1)),
                ("ret-scalar-tmem-y", dict(tb_x=32, tb_y=1, tb_z=4, sd=2, bm_x=1, qstore=2,
                                           prefetch=2, sb=4))]


@pytest.mark.parametrize("name,kw", RHS4_RETIMED, ids=[p[0] for p in RHS4_RETIMED])
def test_rhs4_retimed_ragged(name, kw):
    """rhs4's retimed column walk (R16): outer-s products scattered to the
    pending outputs, inner-s product planes with their halo columns, s-window queue; ragged
    grid (odd nx: the last pair of a row half outside; SB chunks with a ragged tail),
    poisoned far halo, NaN-filled outputs."""
    kind, r = 4, 2
    L = H.layout((37, 22, 19), r + 1)
    c = H.coeffs(kind, r, "random", seed=11)
    ins = H.inputs(kind, L, seed=17, poison_beyond=r)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    kw = dict(kw)
    _, got = run_gpu(kind, r, c, L, ins, S(**dict(dict(sb=8), **kw)))
    for o in range(ost.N_OUT[kind]):
        H.assert_parity(L, got[o], want[o], f"{name} out{o}")
        H.assert_halo_untouched(L, got[o], np.full(L.numel, np.nan))


@pytest.mark.parametrize("n,kw", [((20, 18, 3), dict(tb_x=8, tb_y=8, bm_x=2, sb=1, prefetch=1)),
                                  ((20, 18, 5), dict(tb_x=8, tb_y=8, bm_x=2, sb=2, prefetch=4)),
                                  ((21, 6, 17), dict(tb_x=16, tb_y=1, tb_z=8, sd=2, bm_x=1,
                                                     sb=2, prefetch=2)),
                                  ((17, 17, 9), dict(tb_x=8, tb_y=16, bm_x=2, sb=1, qstore=2,
                                                   prefetch=1))],
                         ids=["sb1-nz3", "sb2-pf4", "y-sb2-ragged", "tmem-sb1-ragged"])
def test_rhs4_retimed_short_chunks(n, kw):
    """Retimed rhs4 edge cases: chunks of 1-2 planes (every step is warm-up or drain but
    one), a 3-plane grid, a ragged y-streamed grid, the TMEM queue at SB 1."""
    kind, r = 4, 2
    L = H.layout(n, r + 1)
    c = H.coeffs(kind, r, "random", seed=21)
    ins = H.inputs(kind, L, seed=23, poison_beyond=r)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    _, got = run_gpu(kind, r, c, L, ins, S(**kw))
    for o in range(3):
        H.assert_parity(L, got[o], want[o], f"{kw} out{o}")
        H.assert_halo_untouched(L, got[o], np.full(L.numel, np.nan))


def test_integer_polynomial_bit_exact():
    """Integer weights and integer data: FMA is exact, so GPU == oracle bit-for-bit."""
    r = 4
    L = H.layout((12, 10, 9), r)
    c = ost.star_laplacian_coeffs(r, integer=True)
    b = np.full(L.numel, np.nan)
    v = L.view(b)
    ax = np.arange(-r, 12 + r, dtype=np.float64)
    ay = np.arange(-r, 10 + r, dtype=np.float64)
    az = np.arange(-r, 9 + r, dtype=np.float64)
    Z, Y, X = np.meshgrid(az, ay, ax, indexing="ij")
    v[...] = X ** 4 + 3 * Y ** 3 - Z ** 2 * X
    _, want = H.oracle_outputs(1, r, c, L, [b])
    for name, s in [("tma", S(tb_x=8, tb_y=4, sb=4)), ("gather", S(tb_x=8, tb_y=4, sb=4, use_retiming=1)),
                    ("tile", S(tb_x=8, tb_y=2, tb_z=2, staging=2, **NOSTREAM))]:
        _, got = run_gpu(1, r, c, L, [b], s)
        assert np.array_equal(H.interior(L, got[0]), H.interior(L, want[0])), name


@pytest.mark.parametrize("nsteps", [2, 3])
def test_multistep_ping_pong(nsteps):
    kind, r = 1, 2
    L = H.layout((40, 20, 24), r)
    c = H.coeffs(kind, r, "random", seed=7)
    ins = H.inputs(kind, L, seed=9)
    out0 = [ins[0].copy()]
    H.interior(L, out0[0])[...] = np.nan
    win, wout = H.oracle_outputs(kind, r, c, L, ins, nsteps=nsteps)
    gin, gout = run_gpu(kind, r, c, L, ins, S(), nsteps=nsteps, out_init=out0)
    res_g, res_w = (gout[0], wout[0]) if nsteps % 2 else (gin[0], win[0])
    H.assert_parity(L, res_g, res_w, f"T={nsteps}")


def test_device_generator_bit_identical_to_cstgen():
    L = H.layout((37, 19, 11), 3)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    t = torch.empty(L.numel, dtype=torch.float64, device="cuda")
    for z0, nyg, nxg in [(0, None, None), (40, 19, 37)]:
        C.cst_fill_uniform(g, t.data_ptr(), 77, 5, nxg, nyg, z0, float("nan"))
        torch.cuda.synchronize()
        want = cstgen.fill(L, seed=77, array_id=5, z0=z0)
        got = t.cpu().numpy()
        assert np.array_equal(got.view(np.uint64), want.view(np.uint64))


def test_host_path_matches_device_path():
    kind, r = 1, 4
    L = H.layout((48, 40, 36), r)
    c = H.coeffs(kind, r)
    ins = H.inputs(kind, L, seed=4)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    s = C.cst_setting_default(h)
    hin = [torch.from_numpy(ins[0].copy()).pin_memory()]
    hout = [torch.full((L.numel,), float("nan"), dtype=torch.float64).pin_memory()]
    C.cst_sweep_host(h, s, [t.data_ptr() for t in hin], [t.data_ptr() for t in hout], 1)
    C.cst_stencil_destroy(h)
    got = hout[0].numpy()
    H.assert_parity(L, got, want[0], "host path")
    H.assert_halo_untouched(L, got, np.full(L.numel, np.nan))


@pytest.mark.parametrize("kind,r,n", [(3, 4, (40, 24, 36)), (4, 2, (37, 22, 40)), (1, 3, (45, 30, 50))],
                         ids=["hypterm", "rhs4", "star-r3"])
def test_host_path_multi_input_poisoned_padding(kind, r, n):
    """cst_sweep_host uploads per row only the columns a kernel can read (interior + even
    x-halo), not the row padding: NaN in everything beyond the radius (the outer halo ring
    and the row padding) of the host inputs cannot reach an output; multi-input kinds, and an
    odd radius (x-halo rounded up to even)."""
    L = H.layout(n, r + 1)
    c = H.coeffs(kind, r, "random", seed=kind + 40)
    ins = H.inputs(kind, L, seed=41, poison_beyond=r)
    for b in ins:  # poison the row padding too
        v = b.reshape(L.nz + 2 * L.halo, L.ny + 2 * L.halo, L.pitch_x)
        v[:, :, :L.lead_x - L.halo] = np.nan
        v[:, :, L.lead_x + L.nx + L.halo:] = np.nan
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    s = C.cst_setting_default(h)
    hin = [torch.from_numpy(b.copy()).pin_memory() for b in ins]
    hout = [torch.full((L.numel,), float("nan"), dtype=torch.float64).pin_memory()
            for _ in range(ost.N_OUT[kind])]
    C.cst_sweep_host(h, s, [t.data_ptr() for t in hin], [t.data_ptr() for t in hout], 1)
    C.cst_stencil_destroy(h)
    for o in range(ost.N_OUT[kind]):
        H.assert_parity(L, hout[o].numpy(), want[o], f"host out{o}")
        H.assert_halo_untouched(L, hout[o].numpy(), np.full(L.numel, np.nan))


def test_invalid_arguments_on_gpu():
    L = H.layout((16, 16, 16), 2)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(1, 2, list(H.coeffs(1, 2)), g)
    t = torch.zeros(L.numel, dtype=torch.float64, device="cuda")
    s = C.cst_setting_default(h)
    with pytest.raises(C.CstError) as e:
        C.cst_sweep(h, s, [t.data_ptr()], [t.data_ptr()])
    assert e.value.status == C.CST_E_INVALID
    t2 = torch.zeros(L.numel, dtype=torch.float64, device="cuda")
    bad = S(tb_x=1024, tb_y=2)
    with pytest.raises(C.CstError) as e:
        C.cst_sweep(h, bad, [t.data_ptr()], [t2.data_ptr()])
    assert e.value.status == C.CST_E_CONSTRAINT
    C.cst_stencil_destroy(h)


def test_host_path_multistep_and_chunked():
    kind, r = 1, 2
    L = H.layout((48, 40, 70), r)                      # 70 planes -> several pipeline chunks
    c = H.coeffs(kind, r, "random", seed=8)
    ins = H.inputs(kind, L, seed=12)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    s = C.cst_setting_default(h)
    # one step, pipelined over z-chunks
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    hin = [torch.from_numpy(ins[0].copy()).pin_memory()]
    hout = [torch.full((L.numel,), float("nan"), dtype=torch.float64).pin_memory()]
    C.cst_sweep_host(h, s, [t.data_ptr() for t in hin], [t.data_ptr() for t in hout], 1)
    assert C.cst_last_launch_count(h) > 1
    H.assert_parity(L, hout[0].numpy(), want[0], "host chunked")
    H.assert_halo_untouched(L, hout[0].numpy(), np.full(L.numel, np.nan))
    # two steps (ping-pong through the host buffers)
    out0 = ins[0].copy()
    H.interior(L, out0)[...] = np.nan
    win, wout = H.oracle_outputs(kind, r, c, L, ins, nsteps=2)
    hin = [torch.from_numpy(ins[0].copy()).pin_memory()]
    hout = [torch.from_numpy(out0).pin_memory()]
    C.cst_sweep_host(h, s, [t.data_ptr() for t in hin], [t.data_ptr() for t in hout], 2)
    H.assert_parity(L, hin[0].numpy(), win[0], "host T=2")
    C.cst_stencil_destroy(h)


# hypterm-like register path over every staging of the fast streaming kernel; the TMA cases
# use the per-array halo layout (q_a: a-halo only, q_b: b-halo only, q_s: none)
HYP_PATHS = [
    ("tma-z-32x4", S(tb_x=32, tb_y=4, sb=8, prefetch=2)),
    ("tma-z-16x8-pf3", S(tb_x=16, tb_y=8, sb=8, prefetch=3)),
    ("tma-z-32x8", S(tb_x=32, tb_y=8, sb=8, prefetch=2)),
    ("tma-y-16x1x8", S(tb_x=16, tb_y=1, tb_z=8, sd=2, sb=8, prefetch=3)),
    ("tma-y-32x1x4-sb16", S(tb_x=32, tb_y=1, tb_z=4, sd=2, sb=16, prefetch=2)),
    ("tma-z-gather", S(tb_x=32, tb_y=4, sb=8, use_retiming=1, prefetch=2)),
    ("tma-z-const-pf4", S(tb_x=16, tb_y=8, sb=8, use_constant=2, prefetch=4)),
    ("ldst-z", S(tb_x=32, tb_y=4, sb=8, staging=2, prefetch=1)),
    ("none-y", S(tb_x=16, tb_y=1, tb_z=8, sd=2, sb=8, staging=1, prefetch=1)),
]


@pytest.mark.parametrize("name,setting", HYP_PATHS, ids=[p[0] for p in HYP_PATHS])
def test_hypterm_paths_ragged(name, setting):
    kind, r = 3, 4
    L = H.layout((37, 29, 26), r + 1)
    c = H.coeffs(kind, r, "random", seed=5)
    ins = H.inputs(kind, L, seed=17, poison_beyond=r)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    _, got = run_gpu(kind, r, c, L, ins, setting)
    for o in range(5):
        H.assert_parity(L, got[o], want[o], f"{name} out{o}")
        H.assert_halo_untouched(L, got[o], np.full(L.numel, np.nan))
