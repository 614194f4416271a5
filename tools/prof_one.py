"""Run one setting a few times at full size (for ncu captures; no parity, no timing).

    python tools/prof_one.py KIND ORDER NXxNYxNZ NSTEPS SETTING_JSON|default|tuned/<file>
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402

kind, r = int(sys.argv[1]), int(sys.argv[2])
n = [int(v) for v in sys.argv[3].split("x")]
nsteps = int(sys.argv[4])
arg = sys.argv[5]
nc = {1: 6 * r + 1, 2: 27, 3: 7, 4: 3}[kind]
g = C.make_grid(*n, r)
h = C.cst_stencil_create(kind, r, [0.1] * nc if kind < 3 else ([4 / 5, -1 / 5, 4 / 105, -1 / 280, 1, 1, 1] if kind == 3 else [1, 1, 1]), g)
if arg == "default":
    s = C.cst_setting_default(h)
elif arg.endswith(".json") and os.path.exists(os.path.join(ROOT, arg)):
    s = C.cst_setting.from_dict(json.load(open(os.path.join(ROOT, arg)))["setting"])
else:  # partial dicts are completed from explore.py's base setting
    d = dict(tb_x=64, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=128,
             uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=1, bm_y=1, bm_z=1,
             use_retiming=2, prefetch=3, bt=1)
    d.update(json.loads(arg))
    s = C.cst_setting.from_dict(d)
ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_IN[kind])]
outs = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_OUT[kind])]
for a, t in enumerate(ins):
    C.cst_fill_uniform(g, t.data_ptr(), 3, a)
for _ in range(3):
    C.cst_sweep(h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs], nsteps,
                torch.cuda.current_stream().cuda_stream)
C.cst_sync(h)
print("done", s.as_dict())
