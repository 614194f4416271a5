"""Run one setting once on a small grid vs the oracle (debug helper)."""
import json
import sys
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402
import gpu_helpers as H  # noqa: E402
from oracle import stencil as ost  # noqa: E402

kind, r = int(sys.argv[1]), int(sys.argv[2])
n = tuple(int(v) for v in sys.argv[3].split("x"))
d = json.loads(sys.argv[4])
L = H.layout(n, r)
c = H.coeffs(kind, r, "random", seed=1)
ins = H.inputs(kind, L, seed=5)
_, want = H.oracle_outputs(kind, r, c, L, ins)
g = C.cst_grid(L.nx, L.ny, L.nz, L.halo, L.lead_x, L.pitch_x, L.pitch_y)
h = C.cst_stencil_create(kind, r, list(c), g)
s = C.cst_setting_default(h) if d == "default" else C.cst_setting.from_dict(d)
print("setting", s.as_dict(), flush=True)
dins = [torch.from_numpy(b).cuda() for b in ins]
douts = [torch.full((L.numel,), float("nan"), dtype=torch.float64, device="cuda") for _ in want]
C.cst_sweep(h, s, [t.data_ptr() for t in dins], [t.data_ptr() for t in douts], 1,
            torch.cuda.current_stream().cuda_stream)
C.cst_sync(h)
for o, w in zip(douts, want):
    H.assert_parity(L, o.cpu().numpy(), w, "run_one")
print("OK")
