"""Host-path probe: pinned H2D / D2H bandwidth alone and concurrent (torch copies), then
cst_sweep_host of the star25 512^3 bench workload (one step; profiles/r02/g08_e2e_probe.jsonl
and g51_host_chunks.txt have the chunk-count sweeps that set cst_sweep_host's 32 pipeline chunks)."""
import json, os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402
import bench  # noqa: E402

n = 1 << 27                                     # 1 GiB of doubles
h = torch.empty(n, dtype=torch.float64).pin_memory()
h2 = torch.empty(n, dtype=torch.float64).pin_memory()
d = torch.empty(n, dtype=torch.float64, device="cuda")
d2 = torch.empty(n, dtype=torch.float64, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
res = {}
for name, fn in [("h2d", lambda: d.copy_(h, non_blocking=True)),
                 ("d2h", lambda: h.copy_(d, non_blocking=True))]:
    fn(); torch.cuda.synchronize()
    t0 = time.perf_counter(); fn(); torch.cuda.synchronize()
    res[name + "_GBs"] = n * 8 / (time.perf_counter() - t0) / 1e9
torch.cuda.synchronize()
t0 = time.perf_counter()
with torch.cuda.stream(s1):
    d.copy_(h, non_blocking=True)
with torch.cuda.stream(s2):
    h2.copy_(d2, non_blocking=True)
torch.cuda.synchronize()
res["concurrent_each_GBs"] = n * 8 / (time.perf_counter() - t0) / 1e9
del h, h2, d, d2
torch.cuda.empty_cache()
g = C.make_grid(512, 512, 512, 4)
hs = C.cst_stencil_create(1, 4, bench.star_coeffs(), g)
st = C.cst_setting.from_dict(json.load(open(os.path.join(ROOT, "tuned", "star25_512.json")))["setting"])
hu = torch.empty(g.numel, dtype=torch.float64).pin_memory()
hv = torch.empty(g.numel, dtype=torch.float64).pin_memory()
hu.uniform_(-1, 1)
C.cst_sweep_host(hs, st, [hu.data_ptr()], [hv.data_ptr()], 1)
t0 = time.perf_counter()
for _ in range(3):
    C.cst_sweep_host(hs, st, [hu.data_ptr()], [hv.data_ptr()], 1)
res["sweep_host_ms"] = (time.perf_counter() - t0) / 3 * 1e3
print(json.dumps(res))
