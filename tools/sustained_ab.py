"""Sustained-regime A/B timing: the B200 holds its boost clock for
the first ~75 ms of back-to-back sweeps, then the SW power cap lowers the SM clock; kernels
bound by an SM-side pipe (shared memory, FP64) slow down with it.  This tool pre-heats the
GPU with `--heat-ms` of sweeps, then times the given settings interleaved in blocks of
`--block` launches (A B C A B C ...) for `--rounds` rounds, CUDA events per launch on one
stream, NVML SM clock / power sampled every 2 ms.  One JSON line: per setting the mean and
median ms of its sustained blocks, the SM clock median during them, and the burst time (the
setting's first launches after a 300 ms idle, before the heat).

    python tools/sustained_ab.py --config star25 --settings '[{}, {"bm_y": 4, "tb_y": 2}]'
Overrides apply to the tuned setting (tuned/<config>_*.json) or the default.
"""
import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402
import tune  # noqa: E402

TUNED = {"star25": "star25_512.json", "box27": "box27_512.json", "hypterm": "hypterm_512.json",
         "rhs4": "rhs4_320.json"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="star25")
    ap.add_argument("--settings", default="[{}]")
    ap.add_argument("--block", type=int, default=100)
    ap.add_argument("--rounds", type=int, default=6)
    ap.add_argument("--heat-ms", type=float, default=1500.0)
    ap.add_argument("--burst", type=int, default=10)
    ap.add_argument("--isolated", action="store_true",
                    help="each setting alone: cool down --cool-s, then --heat-ms of back-to-back "
                         "sweeps; burst = the first --burst launches, steady = launches after "
                         "--settle-ms")
    ap.add_argument("--cool-s", type=float, default=3.0)
    ap.add_argument("--settle-ms", type=float, default=400.0)
    ap.add_argument("--burst-ab", type=int, default=0,
                    help="burst A/B: this many rounds of (0.5 s idle, 30 launches) per setting, "
                         "settings interleaved; reports the median of the per-round medians")
    a = ap.parse_args()
    kind, r, coeffs, n, seed = tune.config(a.config)
    g = C.make_grid(*n, r)
    h = C.cst_stencil_create(kind, r, coeffs, g)
    ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_IN[kind])]
    outs = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_OUT[kind])]
    for i, t in enumerate(ins):
        C.cst_fill_uniform(g, t.data_ptr(), seed, i)
    p = os.path.join(ROOT, "tuned", TUNED[a.config])
    base = (json.load(open(p))["setting"] if os.path.exists(p)
            else C.cst_setting_default(h).as_dict())
    settings = []
    for ov in json.loads(a.settings):
        d = dict(base, **ov)
        s = C.cst_setting.from_dict(d)
        try:
            C.cst_setting_check(h, s)
            C.cst_kernel_info_get(h, s)        # compile + R13 before any timing
            settings.append((ov, s))
        except C.CstError as e:
            print(json.dumps({"skipped": ov, "why": str(e)}), flush=True)
    ip, op = [t.data_ptr() for t in ins], [t.data_ptr() for t in outs]
    st = torch.cuda.Stream()
    samples, stop = [], threading.Event()

    def poll():
        try:
            import pynvml as nv
            nv.nvmlInit()
            dev = nv.nvmlDeviceGetHandleByIndex(torch.cuda.current_device())
            t0 = time.time()
            while not stop.is_set():
                samples.append((time.time() - t0, nv.nvmlDeviceGetClockInfo(dev, nv.NVML_CLOCK_SM),
                                nv.nvmlDeviceGetPowerUsage(dev) / 1000.0))
                time.sleep(0.002)
        except Exception:  # noqa: BLE001
            pass

    def run(s, k):
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(k + 1)]
        with torch.cuda.stream(st):
            ev[0].record(st)
            for i in range(k):
                C.cst_sweep(h, s, ip, op, 1, st.cuda_stream)
                ev[i + 1].record(st)
        torch.cuda.synchronize()
        return [ev[i].elapsed_time(ev[i + 1]) for i in range(k)]

    if a.burst_ab > 0:
        pts = n[0] * n[1] * n[2]
        bpp = 8 * (C.N_IN[kind] + C.N_OUT[kind])
        per = {json.dumps(ov): [] for ov, _ in settings}
        for _ in range(a.burst_ab):
            for ov, s in settings:
                time.sleep(0.5)
                per[json.dumps(ov)].append(statistics.median(run(s, 30)))
        out = {"config": a.config, "grid": list(n), "mode": "burst_ab", "rounds": a.burst_ab,
               "base": base, "results": []}
        for k, v in per.items():
            m = statistics.median(v)
            out["results"].append({"override": json.loads(k), "round_medians_ms": v,
                                   "median_ms": m, "gstencils": pts / (m * 1e-3) / 1e9,
                                   "alg_GBs": pts * bpp / (m * 1e-3) / 1e9})
        print(json.dumps(out), flush=True)
        C.cst_stencil_destroy(h)
        return
    if a.isolated:
        th = threading.Thread(target=poll, daemon=True)
        th.start()
        t_start = time.time()
        pts = n[0] * n[1] * n[2]
        bpp = 8 * (C.N_IN[kind] + C.N_OUT[kind])
        out = {"config": a.config, "grid": list(n), "mode": "isolated", "heat_ms": a.heat_ms,
               "settle_ms": a.settle_ms, "cool_s": a.cool_s, "base": base, "results": []}
        for ov, s in settings:
            time.sleep(a.cool_s)
            t0 = time.time() - t_start
            ms, el = [], 0.0
            while el < a.heat_ms:
                b = run(s, 20)
                ms += b
                el += sum(b)
            t1 = time.time() - t_start
            cum, steady = 0.0, []
            for m in ms:
                cum += m
                if cum >= a.settle_ms:
                    steady.append(m)
            t_settle = t0 + (t1 - t0) * (a.settle_ms / max(el, 1e-9))
            cl = [c for (t, c, pw) in samples if t_settle <= t <= t1]
            pw = [q for (t, c, q) in samples if t_settle <= t <= t1]
            sm = statistics.mean(steady) if steady else float("nan")
            out["results"].append({
                "override": ov, "launches": len(ms),
                "burst_median_ms": statistics.median(ms[:a.burst]),
                "steady_mean_ms": sm, "steady_gstencils": pts / (sm * 1e-3) / 1e9,
                "steady_alg_GBs": pts * bpp / (sm * 1e-3) / 1e9,
                "steady_sm_clock_median": statistics.median(cl) if cl else None,
                "steady_power_median_W": statistics.median(pw) if pw else None,
                "series_ms_every_20th": [round(m, 4) for m in ms[::20]]})
        stop.set()
        th.join()
        print(json.dumps(out), flush=True)
        C.cst_stencil_destroy(h)
        return
    res = {ov_s: {"burst": [], "sustained": [], "clock": [], "power": []}
           for ov_s in (json.dumps(ov) for ov, _ in settings)}
    th = threading.Thread(target=poll, daemon=True)
    th.start()
    t_start = time.time()
    for ov, s in settings:                     # burst: after an idle gap
        time.sleep(0.3)
        res[json.dumps(ov)]["burst"] = run(s, a.burst)
    # heat with the first setting
    t_heat = time.time()
    while (time.time() - t_heat) * 1e3 < a.heat_ms:
        run(settings[0][1], 50)
    for _ in range(a.rounds):
        for ov, s in settings:
            t0 = time.time() - t_start
            ms = run(s, a.block)
            t1 = time.time() - t_start
            k = json.dumps(ov)
            res[k]["sustained"] += ms
            cl = [c for (t, c, pw) in samples if t0 <= t <= t1]
            pw = [q for (t, c, q) in samples if t0 <= t <= t1]
            res[k]["clock"] += cl
            res[k]["power"] += pw
    stop.set()
    th.join()
    out = {"config": a.config, "grid": list(n), "block": a.block, "rounds": a.rounds,
           "heat_ms": a.heat_ms, "base": base, "results": []}
    pts = n[0] * n[1] * n[2]
    bpp = 8 * (C.N_IN[kind] + C.N_OUT[kind])
    for k, v in res.items():
        sm = statistics.mean(v["sustained"])
        out["results"].append({
            "override": json.loads(k), "burst_median_ms": statistics.median(v["burst"]),
            "sustained_mean_ms": sm, "sustained_median_ms": statistics.median(v["sustained"]),
            "sustained_gstencils": pts / (sm * 1e-3) / 1e9,
            "sustained_alg_GBs": pts * bpp / (sm * 1e-3) / 1e9,
            "sm_clock_median": statistics.median(v["clock"]) if v["clock"] else None,
            "power_median_W": statistics.median(v["power"]) if v["power"] else None})
    print(json.dumps(out), flush=True)
    C.cst_stencil_destroy(h)


if __name__ == "__main__":
    main()
