"""cst_dist_tune on the GPU with its built-in evaluator (code generation of the share on
host threads, CUDA-event timing on this rank's replica): one rank, small grid, short
search.  The result must be a valid setting whose re-timed speed is within the noise of
the reported best, and the report must be consistent (the multi-rank protocol itself is
covered by the gloo tests in test_dist_cpu.py)."""
import pytest

torch = pytest.importorskip("torch")

from cst_testutil import gpu_available  # noqa: E402
import gpu_helpers as H  # noqa: E402
from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402

pytestmark = pytest.mark.gpu
if not gpu_available():
    pytest.skip("no GPU", allow_module_level=True)


def test_dist_tune_single_rank_builtin_evaluator():
    kind, r, n = 1, 2, (96, 64, 64)
    g = C.make_grid(*n, r)
    h = C.cst_stencil_create(kind, r, list(H.coeffs(kind, r)), g)
    u = torch.empty(g.numel, dtype=torch.float64, device="cuda")
    v = torch.empty(g.numel, dtype=torch.float64, device="cuda")
    C.cst_fill_uniform(g, u.data_ptr(), 3, 0)
    o = C.cst_tune_opts_default()
    o.seed = 5
    o.dataset_size = 24
    o.max_generations = 3
    o.time_budget_s = 20
    o.reps = 3
    o.noise_reps = 3
    d = C.cst_dist_create(h, 1, 0, None)
    best, rep = C.cst_dist_tune(d, o, [u.data_ptr()], [v.data_ptr()])
    C.cst_dist_destroy(d)
    C.cst_setting_check(h, best)
    assert rep.evaluations >= 24 and rep.best_ms > 0 and rep.space_count == C.cst_space_count(h)
    assert 0 < rep.sampled_count < rep.space_count
    ms = C.cst_time_setting(h, best, [u.data_ptr()], [v.data_ptr()], 2, 10,
                            torch.cuda.current_stream().cuda_stream)
    assert ms < 1.5 * rep.best_ms + 0.01, (ms, rep.best_ms)
    C.cst_stencil_destroy(h)
