"""crash_sweep.py — random valid settings of the four tuning configs at their full sizes (star25 /
box27 / hypterm 512^3, rhs4 320^3), each swept once on device-generated inputs, to catch faults
the small-grid parity sweeps cannot reach (no oracle at these sizes).

    python tools/crash_sweep.py N_PER_CONFIG SEED
"""
import sys, os, json, random
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, 'tools'))
import torch
from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
import tune
n_per = int(sys.argv[1]); seed = int(sys.argv[2])
for cfg in ('star25', 'box27', 'hypterm', 'rhs4'):
    kind, r, coeffs, n, s0 = tune.config(cfg)
    g = C.make_grid(*n, r)
    h = C.cst_stencil_create(kind, r, coeffs, g)
    ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_IN[kind])]
    outs = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_OUT[kind])]
    for a, t in enumerate(ins): C.cst_fill_uniform(g, t.data_ptr(), s0, a)
    cnt = C.cst_space_count(h)
    rng = random.Random(seed * 7 + kind)
    ok = rej = 0
    for _ in range(n_per):
        s = C.cst_space_at(h, rng.randrange(cnt))
        print(cfg, json.dumps(s.as_dict()), flush=True)
        try:
            C.cst_sweep(h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs], 1, torch.cuda.current_stream().cuda_stream)
            C.cst_sync(h); ok += 1
        except C.CstError as e:
            if e.status == C.CST_E_CONSTRAINT: rej += 1; continue
            print("CULPRIT", cfg, json.dumps(s.as_dict()), str(e), flush=True); sys.exit(3)
    print("RESULT", cfg, ok, rej, flush=True)
    del ins, outs; torch.cuda.empty_cache(); C.cst_stencil_destroy(h)
