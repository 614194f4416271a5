"""z-slab decomposition on one GPU (loopback transport, same code path and halo plan as the
NCCL sweep): the slabs must reproduce the single-grid sweep BIT-IDENTICALLY, for one and
several steps, and match the oracle within 1e-12."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402
import gpu_helpers as H  # noqa: E402
from oracle import stencil as ost  # noqa: E402

pytestmark = pytest.mark.gpu


def S(**kw):
    d = dict(tb_x=32, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=8,
             uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=2, bm_y=2, bm_z=1,
             use_retiming=2, prefetch=2)
    d.update(kw)
    return C.cst_setting.from_dict(d)


SETTINGS = [("tma-retimed", S()), ("tma-gather", S(use_retiming=1, bm_x=1, bm_y=1)),
            ("none", S(staging=1, prefetch=1)),
            ("tile3d", S(use_streaming=1, sd=1, sb=1, prefetch=1, tb_x=16, tb_y=2, tb_z=2,
                         bm_x=1, bm_y=1, staging=2)),
            ("sd-y", S(sd=2, tb_y=1, tb_z=4, bm_y=1, bm_z=1))]


@pytest.mark.parametrize("nslabs", [2, 4])
@pytest.mark.parametrize("nsteps", [1, 2])
@pytest.mark.parametrize("name,s", SETTINGS, ids=[x[0] for x in SETTINGS])
def test_loopback_bit_identical_to_single_grid(nslabs, nsteps, name, s):
    r, nx, ny, nzl, seed = 4, 64, 40, 16, 23
    c = list(H.coeffs(1, r, "random", seed=3))
    gl = C.make_grid(nx, ny, nzl * nslabs, r)
    hg = C.cst_stencil_create(1, r, c, gl)
    ug, vg = [torch.empty(gl.numel, dtype=torch.float64, device="cuda") for _ in range(2)]
    for t in (ug, vg):
        C.cst_fill_uniform(gl, t.data_ptr(), seed, 0)
    C.cst_sweep(hg, s, [ug.data_ptr()], [vg.data_ptr()], nsteps)
    C.cst_sync(hg)
    glob = (vg if nsteps % 2 else ug).cpu().numpy()

    ls = C.make_grid(nx, ny, nzl, r)
    hl = C.cst_stencil_create(1, r, c, ls)
    us = [torch.empty(ls.numel, dtype=torch.float64, device="cuda") for _ in range(nslabs)]
    vs = [torch.empty(ls.numel, dtype=torch.float64, device="cuda") for _ in range(nslabs)]
    for k in range(nslabs):
        for t in (us[k], vs[k]):
            C.cst_fill_uniform(ls, t.data_ptr(), seed, 0, nx, ny, k * nzl)
    C.cst_dist_sweep_loopback(hl, nslabs, s, [t.data_ptr() for t in us], [t.data_ptr() for t in vs],
                              nsteps)
    C.cst_sync(hl)
    assert C.cst_last_launch_count(hl) == nsteps * nslabs * 3
    plane = ls.pitch_y * ls.pitch_x
    for k in range(nslabs):
        res = (vs[k] if nsteps % 2 else us[k]).cpu().numpy()
        a = res[r * plane:(r + nzl) * plane]
        b = glob[(r + k * nzl) * plane:(r + (k + 1) * nzl) * plane]
        ia = a.reshape(nzl, ls.pitch_y, ls.pitch_x)[:, r:r + ny, ls.lead_x:ls.lead_x + nx]
        ib = b.reshape(nzl, ls.pitch_y, ls.pitch_x)[:, r:r + ny, ls.lead_x:ls.lead_x + nx]
        assert np.array_equal(ia.view(np.uint64), ib.view(np.uint64)), (name, k)
    C.cst_stencil_destroy(hg)
    C.cst_stencil_destroy(hl)


def test_loopback_matches_oracle():
    r, n, nslabs = 4, (40, 32, 12), 3
    c = H.coeffs(1, r)
    G = H.layout((n[0], n[1], n[2] * nslabs), r)
    import cstgen
    a = cstgen.fill(G, 5, 0)
    want = np.full(G.numel, np.nan)
    ost.sweep(1, r, c, G, [a], [want])
    ls = C.make_grid(*n, r)
    hl = C.cst_stencil_create(1, r, list(c), ls)
    us = [torch.empty(ls.numel, dtype=torch.float64, device="cuda") for _ in range(nslabs)]
    vs = [torch.full((ls.numel,), float("nan"), dtype=torch.float64, device="cuda")
          for _ in range(nslabs)]
    for k in range(nslabs):
        C.cst_fill_uniform(ls, us[k].data_ptr(), 5, 0, n[0], n[1], k * n[2])
    C.cst_dist_sweep_loopback(hl, nslabs, S(bm_x=1), [t.data_ptr() for t in us],
                              [t.data_ptr() for t in vs], 1)
    C.cst_sync(hl)
    wi = H.interior(G, want)
    scale = np.max(np.abs(wi))
    for k in range(nslabs):
        L = H.layout(n, r)
        got = H.interior(L, vs[k].cpu().numpy())
        err = np.max(np.abs(got - wi[k * n[2]:(k + 1) * n[2]]))
        assert err <= 1e-12 * scale
        # exchanged halo planes hold the neighbour's freshly computed boundary planes
        if k + 1 < nslabs:
            hv = L.view(vs[k].cpu().numpy())[r + n[2]:r + n[2] + r, r:r + n[1], r:r + n[0]]
            nb = H.interior(L, vs[k + 1].cpu().numpy())[:r]
            assert np.array_equal(hv.view(np.uint64), nb.view(np.uint64))
    C.cst_stencil_destroy(hl)
