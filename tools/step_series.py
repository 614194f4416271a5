"""Per-launch time series of the bench's star25 sweep (is the step-time spread periodic,
clustered, or tied to something between launches?). Prints one JSON line."""
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402
import tune  # noqa: E402


def main(n_launch=600, gap_ms=0.0):
    kind, r, coeffs, n, seed = tune.config("star25")
    g = C.make_grid(*n, r)
    h = C.cst_stencil_create(kind, r, coeffs, g)
    u = torch.empty(g.numel, dtype=torch.float64, device="cuda")
    v = torch.empty(g.numel, dtype=torch.float64, device="cuda")
    C.cst_fill_uniform(g, u.data_ptr(), seed, 0)
    s = C.cst_setting.from_dict(json.load(open(os.path.join(ROOT, "tuned", "star25_512.json")))["setting"])
    st = torch.cuda.Stream()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(n_launch + 1)]
    torch.cuda.synchronize()
    samples, stop = [], threading.Event()

    def poll():  # SM / memory clock, power and throttle reasons during the series
        try:
            import pynvml as nv
            nv.nvmlInit()
            dev = nv.nvmlDeviceGetHandleByIndex(torch.cuda.current_device())
            t0 = time.time()
            while not stop.is_set():
                samples.append([round((time.time() - t0) * 1e3, 1),
                                nv.nvmlDeviceGetClockInfo(dev, nv.NVML_CLOCK_SM),
                                nv.nvmlDeviceGetClockInfo(dev, nv.NVML_CLOCK_MEM),
                                nv.nvmlDeviceGetPowerUsage(dev) // 1000,
                                nv.nvmlDeviceGetCurrentClocksEventReasons(dev)])
                time.sleep(0.002)
        except Exception as e:  # noqa: BLE001
            samples.append(str(e))

    th = threading.Thread(target=poll, daemon=True)
    th.start()
    time.sleep(0.02)
    with torch.cuda.stream(st):
        for _ in range(10):
            C.cst_sweep(h, s, [u.data_ptr()], [v.data_ptr()], 1, st.cuda_stream)
        ev[0].record(st)
        for i in range(n_launch):
            C.cst_sweep(h, s, [u.data_ptr()], [v.data_ptr()], 1, st.cuda_stream)
            ev[i + 1].record(st)
    torch.cuda.synchronize()
    stop.set()
    th.join()
    ms = [ev[i].elapsed_time(ev[i + 1]) for i in range(n_launch)]
    med = sorted(ms)[len(ms) // 2]
    slow = [i for i, m in enumerate(ms) if m > 1.1 * med]
    runs, cur = [], 0
    for i in range(n_launch):
        if ms[i] > 1.1 * med:
            cur += 1
        elif cur:
            runs.append(cur)
            cur = 0
    if cur:
        runs.append(cur)
    print(json.dumps({"median": med, "mean": sum(ms) / len(ms), "n_slow": len(slow),
                      "slow_run_lengths": runs, "first_slow": slow[:40],
                      "series": [round(m, 4) for m in ms],
                      "nvml_ms_sm_mem_powerW_reasons": samples}))


if __name__ == "__main__":
    main()
