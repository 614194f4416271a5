"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times: the
same grids, device-generated inputs (same seeds and array ids), coefficients and tuned
settings as bench.py, one cst_sweep, then sampled outputs checked one by one against the
oracle's single-point evaluation on the generator's values at the same global coordinates
(oracle_point_gen).  Samples: uniform random points plus every corner and edge of the
domain, tile boundaries in x and y and the z-chunk boundaries of the setting (SB)."""
import json
import os
import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")

from cst_testutil import ROOT, gpu_available  # noqa: E402
import gpu_helpers as H  # noqa: E402
from oracle import stencil as ost  # noqa: E402
from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402

pytestmark = pytest.mark.gpu
if not gpu_available():
    pytest.skip("no GPU", allow_module_level=True)

# name: (kind, order, grid, seed, coefficients, tuned setting file) — as in bench.py
CONFIGS = {
    "c2_star25_512": (1, 4, (512, 512, 512), 2, ost.star_laplacian_coeffs(4), "star25_512.json"),
    "c1_star13_64": (1, 2, (64, 64, 64), 1, ost.star_laplacian_coeffs(2), None),
    "c3_box27_512": (2, 1, (512, 512, 512), 3, ost.box_binomial_coeffs(), "box27_512.json"),
    "c4_hypterm_512": (3, 4, (512, 512, 512), 4, ost.hypterm_coeffs(), "hypterm_512.json"),
    "next1_rhs4_320": (4, 2, (320, 320, 320), 6, ost.rhs4_coeffs(), "rhs4_320.json"),
}


def samples(n, setting, k=1500, seed=0):
    nx, ny, nz = n
    rng = random.Random(seed)
    pts = {(rng.randrange(nx), rng.randrange(ny), rng.randrange(nz)) for _ in range(k)}
    ex = [0, 1, nx - 2, nx - 1]
    ey = [0, 1, ny - 2, ny - 1]
    ez = [0, 1, nz - 2, nz - 1]
    for x in ex:
        for y in ey:
            for z in ez:
                pts.add((x, y, z))
    tx = setting.tb[0] * setting.bm[0] * setting.cm[0]
    ty = setting.tb[1] * setting.bm[1] * setting.cm[1]
    for t in range(tx, nx, tx):
        for _ in range(2):
            pts.add((t - 1, rng.randrange(ny), rng.randrange(nz)))
            pts.add((t, rng.randrange(ny), rng.randrange(nz)))
    for t in range(ty, ny, ty):
        pts.add((rng.randrange(nx), t - 1, rng.randrange(nz)))
        pts.add((rng.randrange(nx), t, rng.randrange(nz)))
    if setting.use_streaming == 2 and setting.sb > 1:
        for zb in range(setting.sb, nz if setting.sd == 3 else ny, setting.sb):
            for _ in range(4):
                if setting.sd == 3:
                    pts.add((rng.randrange(nx), rng.randrange(ny), zb - 1))
                    pts.add((rng.randrange(nx), rng.randrange(ny), zb))
                else:
                    pts.add((rng.randrange(nx), zb - 1, rng.randrange(nz)))
                    pts.add((rng.randrange(nx), zb, rng.randrange(nz)))
    return sorted(pts)


@pytest.mark.parametrize("name", list(CONFIGS))
def test_full_size_sampled_outputs(name):
    kind, r, n, seed, coeffs, tuned = CONFIGS[name]
    g = C.make_grid(*n, r)
    h = C.cst_stencil_create(kind, r, list(coeffs), g)
    s = C.cst_setting_default(h)
    if tuned:
        s = C.cst_setting.from_dict(json.load(open(os.path.join(ROOT, "tuned", tuned)))["setting"])
    C.cst_setting_check(h, s)
    ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_IN[kind])]
    outs = [torch.full((g.numel,), float("nan"), dtype=torch.float64, device="cuda")
            for _ in range(C.N_OUT[kind])]
    for a, t in enumerate(ins):   # padding beyond the halo poisoned (as bench.py's star25)
        C.cst_fill_uniform(g, t.data_ptr(), seed, a, n[0], n[1], 0, float("nan"))
    C.cst_sweep(h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs], 1,
                torch.cuda.current_stream().cuda_stream)
    C.cst_sync(h)
    pts = samples(n, s, seed=kind)
    idx = torch.tensor([g.offset(x, y, z) for x, y, z in pts], dtype=torch.int64, device="cuda")
    got = np.stack([o.index_select(0, idx).cpu().numpy() for o in outs], axis=1)
    want = np.stack([ost.point_gen(kind, r, coeffs, seed, 0, n[0], n[1], r, x, y, z)
                     for x, y, z in pts])
    assert np.all(np.isfinite(got)), "non-finite output at a sampled point"
    for q in range(C.N_OUT[kind]):
        scale = np.max(np.abs(want[:, q]))
        err = np.max(np.abs(got[:, q] - want[:, q]))
        assert err <= H.TOL * scale, f"{name} out{q}: max err {err:.3e} (scale {scale:.3e})"
    C.cst_stencil_destroy(h)


def test_next2_temporal_blocking_full_size():
    """bench.py's NEXT-2 line: 7-point star, 512^3, 8 steps per call, bt = 2 (fused passes).
    After T steps an output depends on inputs within T*r, so the oracle checks sampled points
    on a local (2Tr+1)^3 box of generator values around each (plain ping-pong; only the
    centre's light cone matters).  Points at least T*r from the boundary."""
    import bench
    import cstgen
    T, r, N, seed = 8, 1, 512, 7
    c = np.array([-6.0] + [1.0, 1.0] * 3)
    g = C.make_grid(N, N, N, r)
    h = C.cst_stencil_create(1, r, list(c), g)
    s = C.cst_setting.from_dict(dict(bench.TBLOCK_SETTING, bt=2))
    u = torch.empty(g.numel, dtype=torch.float64, device="cuda")
    v = torch.empty(g.numel, dtype=torch.float64, device="cuda")
    C.cst_fill_uniform(g, u.data_ptr(), seed, 0)
    C.cst_sweep(h, s, [u.data_ptr()], [v.data_ptr()], T, torch.cuda.current_stream().cuda_stream)
    C.cst_sync(h)
    rng = random.Random(12)
    lo, hi = T * r, N - T * r
    pts = [(rng.randrange(lo, hi), rng.randrange(lo, hi), rng.randrange(lo, hi)) for _ in range(300)]
    pts += [(lo, lo, lo), (hi - 1, hi - 1, hi - 1), (lo, hi - 1, lo)]
    idx = torch.tensor([g.offset(*p) for p in pts], dtype=torch.int64, device="cuda")
    got = u.index_select(0, idx).cpu().numpy()          # T even: result in the input buffer
    m = 2 * (T - 1) * r + 1
    L = cstgen.make_layout(m, m, m, r)
    want = []
    for x, y, z in pts:
        b = np.full(L.numel, np.nan)
        ax = np.arange(-r, m + r) + x - (T - 1) * r
        ay = np.arange(-r, m + r) + y - (T - 1) * r
        az = np.arange(-r, m + r) + z - (T - 1) * r
        Z, Y, X = np.meshgrid(az, ay, ax, indexing="ij")
        L.view(b)[...] = cstgen.at(seed, 0, N, N, r, X, Y, Z)
        ins, outs = [b], [b.copy()]
        ost.sweep(1, r, c, L, ins, outs, nsteps=T, nthreads=1)
        want.append(ins[0][L.offset((T - 1) * r, (T - 1) * r, (T - 1) * r)])
    want = np.array(want)
    assert np.all(np.isfinite(got))
    scale = np.max(np.abs(want))
    assert np.max(np.abs(got - want)) <= H.TOL * scale
    C.cst_stencil_destroy(h)
