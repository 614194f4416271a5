"""random_parity.py — many random valid settings of the newer kernel paths against the oracle
(GPU; a one-off sweep beyond the committed tests): rhs4 retimed settings (use_retiming = 2)
on two ragged grids and hypterm TMEM settings (qstore = 2), NaN-poisoned far halo and
NaN-filled outputs; settings rejected after code generation (R13 spills) are counted.

    python tools/random_parity.py     # one JSON line: ok / constraint / fail
"""
import random, sys, os, json
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), 'tests'))
import numpy as np, torch
from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
import gpu_helpers as H
from oracle import stencil as ost
from test_gpu_sweep import run_gpu
res = {"ok": 0, "constraint": 0, "fail": []}
for kind, r, n, npick, filt in [(4, 2, (37, 22, 19), 80, "ret"), (3, 4, (40, 24, 20), 40, "tmem"), (4, 2, (48, 40, 24), 40, "ret")]:
    L = H.layout(n, r + 1)
    c = H.coeffs(kind, r, "random", seed=kind * 7 + r)
    ins = H.inputs(kind, L, seed=31, poison_beyond=r)
    _, want = H.oracle_outputs(kind, r, c, L, ins)
    g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
    h = C.cst_stencil_create(kind, r, list(c), g)
    cnt = C.cst_space_count(h)
    rng = random.Random(1234 + kind)
    picks = []
    tries = 0
    while len(picks) < npick and tries < 200000:
        tries += 1
        s = C.cst_space_at(h, rng.randrange(cnt))
        d = s.as_dict()
        if filt == "ret" and d["use_retiming"] != 2: continue
        if filt == "tmem" and d["qstore"] != 2: continue
        picks.append(s)
    C.cst_stencil_destroy(h)
    for s in picks:
        try:
            _, got = run_gpu(kind, r, c, L, ins, s)
        except C.CstError as e:
            res["constraint"] += 1
            continue
        try:
            for o in range(ost.N_OUT[kind]):
                H.assert_parity(L, got[o], want[o], "x")
                H.assert_halo_untouched(L, got[o], np.full(L.numel, np.nan))
            res["ok"] += 1
        except AssertionError as e:
            res["fail"].append([kind, s.as_dict(), str(e)[:200]])
print(json.dumps(res))
