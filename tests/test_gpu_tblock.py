"""Temporal blocking (field 20, bt > 1): cst_sweep with fused passes of
bt sweeps vs the oracle's plain ping-pong (oracle/oracle.cpp, nsteps > 1), element by element
on the same cstgen inputs.  Ragged grids (partial tiles in x and y, several z chunks), both
kinds the path supports, bt = 2 and 4, and a poisoned far halo (NaN beyond `order` from the
interior must never reach an interior value)."""
import numpy as np
import pytest
import torch

from cst_testutil import gpu_available
import gpu_helpers as H
from paper_conf_cluster_sunlyjldlq21_b200 import cst as C

pytestmark = pytest.mark.gpu
if not gpu_available():
    pytest.skip("no GPU", allow_module_level=True)


def S(**kw):
    d = dict(tb_x=32, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=16,
             uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=2, bm_y=2, bm_z=1,
             use_retiming=2, prefetch=2, bt=2)
    d.update(kw)
    return C.cst_setting.from_dict(d)


def run(kind, r, c, L, ins, setting, nsteps):
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    try:
        C.cst_setting_check(h, setting)
        din = torch.from_numpy(ins[0].copy()).cuda()
        dout = torch.full((L.numel,), float("nan"), dtype=torch.float64, device="cuda")
        C.cst_sweep(h, setting, [din.data_ptr()], [dout.data_ptr()], nsteps,
                    torch.cuda.current_stream().cuda_stream)
        C.cst_sync(h)
        launches = C.cst_last_launch_count(h)
        return din.cpu().numpy(), dout.cpu().numpy(), launches
    finally:
        C.cst_stencil_destroy(h)


CASES = [
    # kind, r, grid, setting overrides, nsteps, expected kernel passes
    (2, 1, (70, 21, 40), dict(), 4, 2),                         # box, 2 fused passes
    (2, 1, (70, 21, 40), dict(bt=4, bm_y=1, tb_y=8), 8, 2),     # box, bt = 4
    (2, 1, (45, 30, 19), dict(bm_x=1, bm_y=1, prefetch=1), 5, 3),  # odd: 2 + 2 + 1
    (1, 1, (70, 21, 40), dict(), 4, 2),                         # 7-point star
    (1, 2, (66, 26, 33), dict(prefetch=3), 4, 2),               # 13-point star
    (1, 2, (40, 20, 24), dict(bm_x=1, bm_y=1, tb_y=8, bt=4, sb=8), 8, 2),
    (1, 1, (64, 32, 20), dict(bt=4, bm_y=1, tb_y=8), 4, 2),     # 4 steps, bt 4 -> 2 + 2
    (1, 2, (70, 20, 24), dict(), 3, 3),                         # 3 steps -> 1 + 1 + 1
]


@pytest.mark.parametrize("kind,r,n,kw,nsteps,passes", CASES,
                         ids=[f"k{c[0]}r{c[1]}-{c[4]}steps-{i}" for i, c in enumerate(CASES)])
def test_fused_passes_match_oracle_ping_pong(kind, r, n, kw, nsteps, passes):
    L = H.layout(n, r)
    c = H.coeffs(kind, r, "random", seed=3 + nsteps)
    ins = H.inputs(kind, L, seed=21)
    win, wout = H.oracle_outputs(kind, r, c, L, ins, nsteps=nsteps)
    gin, gout, launches = run(kind, r, c, L, ins, S(**kw), nsteps)
    assert launches == passes + 1, f"launches {launches} (passes + halo copy)"
    res_g, res_w = (gout, wout[0]) if nsteps % 2 else (gin, win[0])
    H.assert_parity(L, res_g, res_w, f"bt={kw.get('bt', 2)} T={nsteps}")


def test_far_halo_never_reaches_the_interior():
    kind, r = 2, 1
    L = H.layout((70, 18, 20), 3)                 # halo 3 > order: poison beyond distance 1
    c = H.coeffs(kind, r, "random", seed=5)
    ins = H.inputs(kind, L, seed=8, poison_beyond=r)
    win, _ = H.oracle_outputs(kind, r, c, L, ins, nsteps=4)
    gin, _, _ = run(kind, r, c, L, ins, S(bt=2), 4)
    H.assert_parity(L, gin, win[0], "poisoned far halo")


def test_bt_matches_bt1_bit_for_bit_where_it_should():
    """bt = 1 and bt = 2 settings of the same tile agree to rounding on the interior."""
    kind, r = 1, 2
    L = H.layout((64, 24, 30), r)
    c = H.coeffs(kind, r)
    ins = H.inputs(kind, L, seed=2)
    a, _, _ = run(kind, r, c, L, ins, S(bt=1), 4)
    b, _, _ = run(kind, r, c, L, ins, S(bt=2), 4)
    ia, ib = H.interior(L, a), H.interior(L, b)
    assert np.max(np.abs(ia - ib)) <= H.TOL * np.max(np.abs(ia))


def test_one_step_with_bt_setting_runs_unfused():
    kind, r = 2, 1
    L = H.layout((70, 20, 16), r)
    c = H.coeffs(kind, r)
    ins = H.inputs(kind, L, seed=4)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    _, gout, launches = run(kind, r, c, L, ins, S(bt=2), 1)
    assert launches == 1
    H.assert_parity(L, gout, want[0], "nsteps=1, bt=2")


def test_time_setting_per_step():
    kind, r = 2, 1
    L = H.layout((256, 256, 64), r)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(H.coeffs(kind, r)), g)
    u = torch.zeros(L.numel, dtype=torch.float64, device="cuda")
    v = torch.zeros(L.numel, dtype=torch.float64, device="cuda")
    ms1 = C.cst_time_setting(h, S(bt=1), [u.data_ptr()], [v.data_ptr()], 1, 3, nsteps=4)
    ms2 = C.cst_time_setting(h, S(bt=2), [u.data_ptr()], [v.data_ptr()], 1, 3, nsteps=4)
    assert ms1 > 0 and ms2 > 0
    C.cst_stencil_destroy(h)


def test_tuner_multistep_objective(tmp_path):
    """cst_tune with nsteps = 4 explores bt (field 20) and times per step on its own copies:
    the caller's input is left untouched and the winner reproduces the oracle."""
    kind, r = 1, 1
    L = H.layout((128, 64, 48), r)
    c = H.coeffs(kind, r, "random", seed=2)
    ins = H.inputs(kind, L, seed=3)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    din = torch.from_numpy(ins[0].copy()).cuda()
    dout = torch.full((L.numel,), float("nan"), dtype=torch.float64, device="cuda")
    o = C.cst_tune_opts_default()
    o.seed = 4
    o.dataset_size = 24
    o.max_generations = 3
    o.time_budget_s = 60
    o.reps = 3
    o.nsteps = 4
    o.metrics_mode = 1
    best, rep = C.cst_tune(h, o, [din.data_ptr()], [dout.data_ptr()])
    C.cst_setting_check(h, best)
    assert np.array_equal(din.cpu().numpy(), ins[0], equal_nan=True)   # input untouched
    win, _ = H.oracle_outputs(kind, r, c, L, ins, nsteps=4)
    C.cst_sweep(h, best, [din.data_ptr()], [dout.data_ptr()], 4,
                torch.cuda.current_stream().cuda_stream)
    C.cst_sync(h)
    H.assert_parity(L, din.cpu().numpy(), win[0], f"tuned bt={best.bt}")
    C.cst_stencil_destroy(h)
