"""Run every kernel path once on a small ragged grid (checked against the oracle), for
compute-sanitizer:

    compute-sanitizer --tool memcheck   --error-exitcode 9 python tools/sanitize.py
    compute-sanitizer --tool racecheck  --error-exitcode 9 python tools/sanitize.py
    compute-sanitizer --tool synccheck  --error-exitcode 9 python tools/sanitize.py

Paths: star / box fast streaming with TMA ring (retimed, gather), ld/st and no staging;
y-streaming; generic (T_SD > 1) ring; 3-D tiles; TMEM streamed state (star, hypterm with
two points along b); hypterm register path; rhs4 generic and retimed (ring, register queue,
TMEM queue); temporal blocking (bt = 2, 4 steps); multi-step ping-pong.  The two-process peer-memory twin (CST_REMOTE) runs under
--target-processes all through tests/test_gpu_p2p.py.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402
import gpu_helpers as H  # noqa: E402

BASE = dict(tb_x=32, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=8,
            uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=2, bm_y=2, bm_z=1,
            use_retiming=2, prefetch=2, bt=1, qstore=1)
NOSTREAM = dict(use_streaming=1, sd=1, sb=1, prefetch=1)
# name, kind, r, grid, overrides, nsteps
CASES = [
    ("star4-tma-retimed", 1, 4, (70, 29, 23), dict(prefetch=3), 1),
    ("star4-tma-gather", 1, 4, (70, 29, 23), dict(use_retiming=1), 1),
    ("star4-ldst", 1, 4, (70, 29, 23), dict(staging=2), 1),
    ("star4-none", 1, 4, (70, 29, 23), dict(staging=1, prefetch=1), 1),
    ("star2-ystream", 1, 2, (70, 29, 23), dict(tb_y=1, tb_z=4, sd=2, bm_y=1, bm_z=2), 1),
    ("star2-generic", 1, 2, (37, 29, 23), dict(tb_y=2, tb_z=2, bm_x=1, bm_y=1), 1),
    ("star2-tile3d", 1, 2, (37, 29, 23), dict(tb_x=16, tb_y=2, tb_z=2, bm_x=1, bm_y=1,
                                             **NOSTREAM), 1),
    ("star4-tmem", 1, 4, (70, 29, 23), dict(qstore=2), 1),
    ("star2-multistep", 1, 2, (70, 29, 23), dict(), 3),
    ("star1-tblock-bt2", 1, 1, (70, 30, 19), dict(bt=2, sb=16), 4),
    ("box-tma", 2, 1, (70, 29, 23), dict(), 1),
    ("box-tblock-bt2", 2, 1, (70, 30, 19), dict(bt=2, sb=16), 4),
    ("hyp-tmem-bmy2", 3, 4, (37, 29, 26), dict(bm_x=1, bm_y=2, qstore=2, use_constant=2,
                                               prefetch=3), 1),
    ("hyp-reg-tma", 3, 4, (37, 29, 26), dict(bm_x=1, bm_y=1), 1),
    ("hyp-reg-ldst", 3, 4, (37, 29, 26), dict(bm_x=1, bm_y=1, staging=2, prefetch=1), 1),
    ("rhs4-generic", 4, 2, (37, 22, 19), dict(tb_x=16, tb_y=8, bm_x=1, bm_y=1,
                                              use_retiming=1), 1),
    ("rhs4-paired", 4, 2, (37, 22, 19), dict(tb_x=8, tb_y=8, bm_x=2, bm_y=1,
                                             use_retiming=1), 1),
    # rhs4 retimed column walk (round 2): product planes + one barrier per plane, ring of
    # 2r + PF planes; s-window from the ring (pair), register queue (scalar), TMEM (qstore 2)
    ("rhs4-ret-pair", 4, 2, (37, 22, 19), dict(tb_x=8, tb_y=16, bm_x=2, bm_y=1, prefetch=1,
                                               use_constant=2), 1),
    ("rhs4-ret-scalar", 4, 2, (37, 22, 19), dict(tb_x=16, tb_y=8, bm_x=1, bm_y=1), 1),
    ("rhs4-ret-tmem-256", 4, 2, (37, 22, 19), dict(tb_x=16, tb_y=16, bm_x=2, bm_y=1,
                                                   prefetch=1, qstore=2), 1),
]


def run(name, kind, r, n, over, nsteps):
    L = H.layout(n, r + 1)
    c = H.coeffs(kind, r, "random", seed=3)
    ins = H.inputs(kind, L, seed=7, poison_beyond=r)
    if nsteps > 1:
        ins = H.inputs(kind, L, seed=7)
    win, want = H.oracle_outputs(kind, r, c, L, ins, nsteps=nsteps)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    s = C.cst_setting.from_dict(dict(BASE, **over))
    C.cst_setting_check(h, s)
    dins = [torch.from_numpy(b.copy()).cuda() for b in ins]
    # NaN-filled outputs: a multi-step sweep first copies in[]'s halo into them (Q23)
    douts = [torch.full((L.numel,), float("nan"), dtype=torch.float64, device="cuda")
             for _ in want]
    C.cst_sweep(h, s, [t.data_ptr() for t in dins], [t.data_ptr() for t in douts], nsteps,
                torch.cuda.current_stream().cuda_stream)
    C.cst_sync(h)
    res, ref = (douts, want) if nsteps % 2 else (dins, win)
    for o, w in zip(res, ref):
        H.assert_parity(L, o.cpu().numpy(), w, name)
    C.cst_stencil_destroy(h)
    print("OK", name, flush=True)


if __name__ == "__main__":
    only = sys.argv[1:] or None
    for case in CASES:
        if only is None or case[0] in only:
            run(*case)
    print("ALL OK", flush=True)
