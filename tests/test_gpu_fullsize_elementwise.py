"""Element-by-element parity at the bench's exact settings (VERDICT r1 "weak" #4).

star25 and box27 at BASELINE's full 512^3 with their tuned settings (tuned/*.json, the
launch configuration bench.py times), and the hypterm-like and rhs4-like tuned settings on
64 x 64 x 512 grids (several SB chunks along z, several tiles in x and y): the device
generator fills the inputs (as in bench.py, padding beyond the halo poisoned with NaN),
one cst_sweep, then the inputs are copied to the host, the oracle (oracle/oracle.cpp, all
host cores) sweeps the same buffers, and EVERY interior output is compared with the 1e-12
max-norm rule; output halos must stay untouched (NaN-filled before the sweep)."""
import json
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

from cst_testutil import ROOT, gpu_available  # noqa: E402
import cstgen  # noqa: E402
import gpu_helpers as H  # noqa: E402
from oracle import stencil as ost  # noqa: E402
from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402

pytestmark = pytest.mark.gpu
if not gpu_available():
    pytest.skip("no GPU", allow_module_level=True)

CASES = {
    "c2_star25_512": (1, 4, (512, 512, 512), 2, ost.star_laplacian_coeffs(4), "star25_512.json"),
    "c3_box27_512": (2, 1, (512, 512, 512), 3, ost.box_binomial_coeffs(), "box27_512.json"),
    "c4_hypterm_64x64x512": (3, 4, (64, 64, 512), 4, ost.hypterm_coeffs(), "hypterm_512.json"),
    "next1_rhs4_64x64x512": (4, 2, (64, 64, 512), 6, ost.rhs4_coeffs(), "rhs4_320.json"),
}


@pytest.mark.parametrize("name", list(CASES))
def test_tuned_setting_every_output_matches_oracle(name):
    kind, r, n, seed, coeffs, tuned = CASES[name]
    g = C.make_grid(*n, r)
    L = cstgen.make_layout(*n, r)
    assert (L.pitch_x, L.pitch_y, L.lead_x) == (g.pitch_x, g.pitch_y, g.lead_x)
    s = C.cst_setting.from_dict(json.load(open(os.path.join(ROOT, "tuned", tuned)))["setting"])
    h = C.cst_stencil_create(kind, r, list(coeffs), g)
    C.cst_setting_check(h, s)
    if s.use_streaming == 2:
        ns = n[2] if s.sd == 3 else n[1]
        assert ns // s.sb >= 2, "fewer than 2 SB chunks"
    ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_IN[kind])]
    outs = [torch.full((g.numel,), float("nan"), dtype=torch.float64, device="cuda")
            for _ in range(C.N_OUT[kind])]
    for a, t in enumerate(ins):
        C.cst_fill_uniform(g, t.data_ptr(), seed, a, n[0], n[1], 0, float("nan"))
    C.cst_sweep(h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs], 1,
                torch.cuda.current_stream().cuda_stream)
    C.cst_sync(h)
    C.cst_stencil_destroy(h)
    hin = [t.cpu().numpy() for t in ins]
    del ins
    want = [np.full(L.numel, np.nan) for _ in range(C.N_OUT[kind])]
    ost.sweep(kind, r, coeffs, L, hin, want)
    del hin
    for q, t in enumerate(outs):
        got = t.cpu().numpy()
        H.assert_parity(L, got, want[q], f"{name} out{q}")
        H.assert_halo_untouched(L, got, np.full(L.numel, np.nan))
    del outs
    torch.cuda.empty_cache()
