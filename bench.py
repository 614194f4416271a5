"""bench.py — GStencil/s of the complex-stencil sweep on B200 (BASELINE.json configs[1]).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl cst|reference]

N=1 workload: order-4 25-point star (FD Laplacian, weights /5040), 512^3 FP64 interior,
halo 4, the tuned setting from tuned/star25_512.json (cst_tune output, then the A/B-checked
hill climb of tools/tune.py --refine-all; the default setting if absent).  A step = one sweep (one kernel launch) over inputs resident in HBM; the two
1.18 GB arrays exceed the 126 MB L2, so no flush is needed between steps.
N>1 (torchrun, one rank per GPU): BASELINE configs[4] — the order-4 star on a z-slab
decomposed 1024 x 1024 grid with a 4-plane halo exchange per step.  Headline = WEAK scaling,
256 x 1024 x 1024 per rank (global nz = 256 N), NCCL send/recv overlapped with the interior
(north_star); value = all ranks' points / max-over-ranks device time.  The same line carries
"strong" (the 2048 x 1024 x 1024 grid, 2048/N planes per rank), "p2p" (weak scaling with the
fused peer-memory halo stores) and "population_eval" (configs[4]'s GA part:
evaluations/s of one 32-candidate generation spread round-robin over the N GPUs, C5c).  At
N=1 the same three single-GPU baselines appear in other_configs (c5_weak_slab_1gpu,
c5_strong_1gpu, c5c_population_eval_g1), so E(N) can be formed from either line.

Extra keys: roofline (dominant kernel = the sweep), cpu_baseline (the oracle on a bounded
sample, rank 0 at N=1), e2e (cst_sweep_host: H2D + sweep + D2H through the C ABI), clocks
(NVML polled every 2 ms during the timed region, nvidia-smi as fallback), gpu_launches,
other_configs (configs[0], [2], [3] and the NEXT rows, reported beside the headline).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

BASE = json.load(open(os.path.join(ROOT, "BASELINE.json")))
METRIC = BASE["metric"]
UNIT = "GStencil/s"
N = 512
R = 4
SEED = 2
D2_R4 = [-9, 128, -1008, 8064, -14350, 8064, -1008, 128, -9]


def star_coeffs():
    w = [v / 5040.0 for v in D2_R4]
    side = w[:R] + w[R + 1:]
    return [3 * w[R]] + side * 3


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def load_setting(C, h):
    p = os.path.join(ROOT, "tuned", "star25_512.json")
    if os.path.exists(p):
        d = json.load(open(p))
        s = C.cst_setting.from_dict(d["setting"])
        C.cst_setting_check(h, s)
        return s, "tuned/star25_512.json"
    return C.cst_setting_default(h), "cst_setting_default"


class ClockSampler:
    """SM clock + throttle reasons sampled DURING the timed region: NVML polled every
    ~2 ms from a thread (nvidia-smi's 100 ms loop as a fallback)."""
    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self.stop_flag = threading.Event()
        self.thread = None
        self.proc = None
        self.rows = []
        self.poll_s = float(os.environ.get("CST_BENCH_CLOCK_POLL_MS", "2")) / 1e3

    def start(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)

            def poll():
                while not self.stop_flag.is_set():
                    try:
                        self.samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                        r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                        for n, bit in self.REASONS.items():
                            if r & bit:
                                self.reasons.add(n)
                    except Exception:
                        pass
                    time.sleep(self.poll_s)
            self.thread = threading.Thread(target=poll, daemon=True)
            self.thread.start()
            self.source = "nvml"
        except Exception:
            self.source = "nvidia-smi"
            try:
                self.proc = subprocess.Popen(
                    ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,"
                     "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                     "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                     "--format=csv,noheader,nounits", "-lms", "100"],
                    stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
                self.thread = threading.Thread(target=self._read, daemon=True)
                self.thread.start()
            except Exception:
                self.proc = None

    def _read(self):
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.proc.stdout:
            r = [x.strip() for x in line.split(",")]
            if len(r) >= 6 and r[0].replace(".", "").isdigit():
                self.samples.append(float(r[0]))
                self.max_mhz = float(r[1])
                for n, v in zip(names, r[2:6]):
                    if v.lower() == "active":
                        self.reasons.add(n)

    def stop(self):
        self.stop_flag.set()
        if self.proc is not None:
            time.sleep(0.15)
            self.proc.terminate()
        if self.thread is not None:
            self.thread.join(timeout=2)
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples), "source": self.source}


def ncu_traffic():
    p = os.path.join(ROOT, "profiles", "ncu_star25_512.json")
    if os.path.exists(p):
        try:
            d = json.load(open(p))
            return d.get("dram_bytes_per_launch")
        except Exception:
            return None
    return None


OTHER = {
    # name: (kind, order, coefficients, grid, seed, description)
    "c1_star13_64": (1, 2, None, (64, 64, 64), 1,
                     "configs[0]: order-2 13-point star, 64^3, fixed default setting (L2-resident)"),
    "c3_box27_512": (2, 1, None, (512, 512, 512), 3,
                     "configs[2]: 27-point box (binomial), 512^3, TMA halo staging"),
    "c4_hypterm_512": (3, 4, None, (512, 512, 512), 4,
                       "configs[3]: hypterm-like, 8 in / 5 out, order 4, 512^3"),
    "next1_rhs4_320": (4, 2, None, (320, 320, 320), 6,
                       "SURVEY NEXT-1: rhs4center-like (5 in / 3 out, order 2, 666 FLOPs/pt), "
                       "320^3 as in Table III — FP64-bound"),
}
FLOPS_PER_POINT = {1: None, 2: 53, 3: 358, 4: 666}
FP64_PEAK_SOURCE = ("cst_fp64_peak: DFMA-chain microbenchmark on this GPU (csrc/runtime/peak.cu); "
                    "MEASURED_PEAKS.json has no FP64 figure")
COUNTER_KEY = {"c3_box27_512": "box27", "c4_hypterm_512": "hypterm", "next1_rhs4_320": "rhs4"}


def fp64_from_counters(key, pts, ms, fp64_peak):
    """FP64 fraction from ncu instruction counts: executed FP64 FLOPs per point
    = 2 DFMA + DADD + DMUL from profiles/r02_fp64_counts.json (one ncu launch of the same
    tuned setting), times the points, over this run's CUDA-event time."""
    p = os.path.join(ROOT, "profiles", "r02_fp64_counts.json")
    if not key or not fp64_peak or not os.path.exists(p):
        return {}
    try:
        d = json.load(open(p))[key]
    except (KeyError, ValueError):
        return {}
    ex = d["executed_fp64_flops_per_point"]
    tf = pts * ex / (ms * 1e-3) / 1e12
    return {"fp64_executed_flops_per_point_ncu": ex, "achieved_TFLOPs_executed": tf,
            "fp64_frac_counters": tf / fp64_peak, "fp64_counts_source": "profiles/r02_fp64_counts.json"}


def other_coeffs(kind, r):
    if kind == 1:
        w = {2: [-1 / 12, 16 / 12, -30 / 12, 16 / 12, -1 / 12]}[r]
        return [3 * w[r]] + (w[:r] + w[r + 1:]) * 3
    if kind == 2:
        b = [0.25, 0.5, 0.25]
        return [x * y * z for x in b for y in b for z in b]
    if kind == 4:
        return [1.0, 1.0, 1.0]
    return [4 / 5, -1 / 5, 4 / 105, -1 / 280, 1.0, 1.0, 1.0]


OTHER_COOL_S = 2.0


def other_configs(C, torch, peak, steps=10, fp64_peak=None, cool_s=OTHER_COOL_S):
    """The other single-GPU configs of BASELINE.json, each timed the same way (CUDA events,
    inputs resident, device generator), with their own roofline fractions.  Each is timed
    after `cool_s` of GPU idle, so that it runs in the burst regime like the headline (which
    runs first, on a cool GPU) rather than under the board power cap that the preceding
    sustained and e2e runs leave behind (power-state-consistent evaluation)."""
    res = {}
    for name, (kind, r, _, n, seed, desc) in OTHER.items():
        g = C.make_grid(*n, r)
        h = C.cst_stencil_create(kind, r, other_coeffs(kind, r), g)
        tuned = os.path.join(ROOT, "tuned", {"c3_box27_512": "box27_512.json",
                                             "c4_hypterm_512": "hypterm_512.json",
                                             "next1_rhs4_320": "rhs4_320.json"}.get(name, "-"))
        src = "cst_setting_default"
        s = C.cst_setting_default(h)
        if os.path.exists(tuned):
            try:
                t = C.cst_setting.from_dict(json.load(open(tuned))["setting"])
                C.cst_setting_check(h, t)
                s, src = t, os.path.relpath(tuned, ROOT)
            except Exception:
                pass
        ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_IN[kind])]
        outs = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_OUT[kind])]
        for a, t in enumerate(ins):
            C.cst_fill_uniform(g, t.data_ptr(), seed, a)
        C.cst_variant_compile(h, s)  # JIT outside the cool-down
        torch.cuda.synchronize()
        time.sleep(cool_s)
        ms = C.cst_time_setting(h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs],
                                3, steps, torch.cuda.current_stream().cuda_stream)
        pts = n[0] * n[1] * n[2]
        bpp = 8 * (C.N_IN[kind] + C.N_OUT[kind])
        gbs = pts * bpp / (ms * 1e-3) / 1e9
        res[name] = {"workload": desc, "gstencils": pts / (ms * 1e-3) / 1e9, "ms_median": ms,
                     "alg_bytes_per_point": bpp, "achieved_GBs": gbs,
                     "hbm_frac_measured": None if n[0] < 128 else gbs / peak,
                     "hbm_frac_nominal_8TBs": None if n[0] < 128 else gbs / 8000.0,
                     "setting": s.as_dict(), "setting_source": src,
                     "timed_after_idle_s": cool_s}
        fpp = FLOPS_PER_POINT.get(kind)
        if fpp and fp64_peak:
            tf = pts * fpp / (ms * 1e-3) / 1e12
            res[name].update({"flops_per_point_as_written": fpp, "achieved_TFLOPs": tf,
                              "fp64_frac_measured": tf / fp64_peak,
                              "fp64_peak_source": FP64_PEAK_SOURCE})
        res[name].update(fp64_from_counters(COUNTER_KEY.get(name), pts, ms, fp64_peak))
        del ins, outs
        C.cst_stencil_destroy(h)
        torch.cuda.empty_cache()
    return res


TBLOCK_SETTING = dict(tb_x=32, tb_y=8, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3,
                      sb=128, uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=2, bm_y=2,
                      bm_z=1, use_retiming=2, prefetch=2)


def tblock_config(C, torch, peak, nsteps=8, steps=5):
    """temporal blocking.  8 ping-pong steps of the order-1 (7-point) star at
    512^3 per cst_sweep call, ms per step, with the fused bt = 2 setting (measured best,
    profiles/r01_tblock_explore.json) against the same tile unfused (bt = 1).  Algorithmic
    HBM bytes per step = 16 B / bt per point."""
    n, r = (512, 512, 512), 1
    g = C.make_grid(*n, r)
    w = [1.0, -2.0, 1.0]
    h = C.cst_stencil_create(1, r, [3 * w[1]] + [w[0], w[2]] * 3, g)
    ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda")]
    outs = [torch.empty(g.numel, dtype=torch.float64, device="cuda")]
    pts = n[0] * n[1] * n[2]
    res = {"workload": "SURVEY NEXT-2: 7-point star (order 1), 512^3, 8 steps per call, "
                       "temporal blocking bt=2 vs bt=1 (ms per step)", "nsteps": nsteps}
    for bt in (1, 2):
        s = C.cst_setting.from_dict(dict(TBLOCK_SETTING, bt=bt))
        C.cst_fill_uniform(g, ins[0].data_ptr(), 7, 0)
        ms = C.cst_time_setting(h, s, [ins[0].data_ptr()], [outs[0].data_ptr()], 2, steps,
                                torch.cuda.current_stream().cuda_stream, nsteps=nsteps)
        gbs = pts * 16.0 / bt / (ms * 1e-3) / 1e9
        res[f"bt{bt}"] = {"gstencils_per_step": pts / (ms * 1e-3) / 1e9, "ms_per_step": ms,
                          "alg_hbm_bytes_per_point_step": 16.0 / bt, "achieved_GBs": gbs,
                          "hbm_frac_measured": gbs / peak, "setting": s.as_dict()}
    res["speedup_bt2_over_bt1"] = res["bt2"]["gstencils_per_step"] / res["bt1"]["gstencils_per_step"]
    del ins, outs
    C.cst_stencil_destroy(h)
    torch.cuda.empty_cache()
    return res


def cpu_baseline(target_s: float = 10.0):
    """The oracle, as it stands, on a bounded sample of the same workload: a 512 x 512 x 16
    slab of the 512^3 star25 grid swept repeatedly until >= target_s seconds."""
    import numpy as np

    import cstgen
    from oracle import stencil as ost
    nz_s = 16
    L = cstgen.make_layout(N, N, nz_s, R)
    u = cstgen.fill(L, SEED, 0)
    v = np.full(L.numel, np.nan)
    c = ost.star_laplacian_coeffs(R)
    cores = os.cpu_count() or 1
    pts, t0 = 0, time.perf_counter()
    while True:
        ost.sweep(1, R, c, L, [u], [v], nthreads=cores)
        pts += N * N * nz_s
        el = time.perf_counter() - t0
        if el >= target_s:
            break
    t1 = time.perf_counter()                       # and once on a single thread
    ost.sweep(1, R, c, L, [u], [v], nthreads=1)
    single = N * N * nz_s / (time.perf_counter() - t1) / 1e9
    cpu_model = ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                cpu_model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"value": pts / el / 1e9, "unit": UNIT, "cores": cores, "kind": "oracle",
            "single_thread_value": single, "cpu_model": cpu_model,
            "sample": f"{N}x{N}x{nz_s} slab of the 512^3 star25 workload, swept "
                      f"{pts // (N * N * nz_s)} times ({el:.1f} s, {cores} OpenMP threads)"}


def run_reference(args, rank, world):
    """--impl reference: the oracle (CPU) timed on the box's host cores, rank 0 only."""
    if rank != 0:
        return
    import numpy as np

    import cstgen
    from oracle import stencil as ost
    nz_s = 8
    L = cstgen.make_layout(N, N, nz_s, R)
    u = cstgen.fill(L, SEED, 0)
    v = np.full(L.numel, np.nan)
    c = ost.star_laplacian_coeffs(R)
    cores = os.cpu_count() or 1
    for _ in range(args.warmup):
        ost.sweep(1, R, c, L, [u], [v], nthreads=cores)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        ost.sweep(1, R, c, L, [u], [v], nthreads=cores)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    pts = N * N * nz_s * args.steps
    val = pts / tot / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (cstgen splitmix64 U[-1,1), seed 2)",
            "config": {"workload": "star25 (order-4 25-point star FD Laplacian) 512^3 FP64 "
                                   "(BASELINE configs[1]); each step a bounded 512x512x8 slab"},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": f"{N}x{N}x{nz_s} slab per step"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------------- configs[4]
C5_NXY, C5_WEAK_NZ, C5_STRONG_NZ, C5_SEED = 1024, 256, 2048, 5


def _gather(dist, world, x):
    """Every rank's x (all ranks, rank order); [x] on one process."""
    if world == 1:
        return [x]
    out = [None] * world
    dist.all_gather_object(out, x)
    return out


def c5_setting(C, h):
    """The tuned star25 setting (tuned/star25_512.json) if valid on this slab, else the
    library default."""
    try:
        s, src = load_setting(C, h)
        return s, src
    except C.CstError:
        return C.cst_setting_default(h), "cst_setting_default"


def c5_sweep(C, torch, dist, rank, world, local, nzl, transport, steps, warmup, peak):
    """One z-slab sweep series of configs[4] (star25, 1024 x 1024 planes, nzl local planes
    per rank): `warmup` + `steps` single-step cst_dist_sweep calls (cst_sweep at world 1),
    CUDA events per step on the sweep stream, total time = max over ranks.  Returns the
    rank-0 view (aggregate GSt/s, per-rank roofline) or None where the transport could
    not be set up (reason given)."""
    g = C.make_grid(C5_NXY, C5_NXY, nzl, R)
    h = C.cst_stencil_create(C.CST_STAR, R, star_coeffs(), g, local)
    s, s_src = c5_setting(C, h)
    u = torch.empty(g.numel, dtype=torch.float64, device="cuda")
    v = torch.empty(g.numel, dtype=torch.float64, device="cuda")
    stream = torch.cuda.current_stream()
    for t in (u, v):
        C.cst_fill_uniform(g, t.data_ptr(), C5_SEED, 0, C5_NXY, C5_NXY, rank * nzl,
                           float("nan"), stream.cuda_stream)
    d, why = None, ""
    if world > 1 and transport == "nccl":
        uid = C.cst_dist_nccl_unique_id() if rank == 0 else None
        obj = [uid]
        dist.broadcast_object_list(obj, src=0)
        d = C.cst_dist_create(h, world, rank, obj[0])
    elif world > 1:
        # every rank must take the same transport: export, all-gather, import, MIN-agree
        d = C.cst_dist_create(h, world, rank, None)
        ok, mine = True, None
        try:
            mine = C.cst_dist_p2p_export(d, [u.data_ptr()], [v.data_ptr()])
        except C.CstError as e:
            ok, why = False, str(e)
        blobs = [None] * world
        dist.all_gather_object(blobs, (ok, mine))
        if ok and all(b[0] for b in blobs):
            try:
                for peer in (rank - 1, rank + 1):
                    if 0 <= peer < world:
                        C.cst_dist_p2p_import(d, peer, blobs[peer][1])
            except C.CstError as e:
                ok, why = False, str(e)
        else:
            ok, why = False, why or "a peer could not export"
        if not all(_gather(dist, world, ok)):
            C.cst_dist_destroy(d)
            C.cst_stencil_destroy(h)
            return {"unavailable": "p2p setup failed: " + (why or "on another rank")[:160]}
    bufs = [u, v]

    def step(i):
        a, b = bufs[i % 2], bufs[1 - i % 2]
        if d is not None:
            C.cst_dist_sweep(d, s, [a.data_ptr()], [b.data_ptr()], 1, stream.cuda_stream)
        else:
            C.cst_sweep(h, s, [a.data_ptr()], [b.data_ptr()], 1, stream.cuda_stream)

    for i in range(max(warmup, 3)):
        step(i)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(steps + 1)]
    evs[0].record(stream)
    launches = 0
    for i in range(steps):
        step(i)
        launches += C.cst_last_launch_count(h)
        evs[i + 1].record(stream)
    torch.cuda.synchronize()
    per = [evs[i].elapsed_time(evs[i + 1]) for i in range(steps)]
    mine_ms = evs[0].elapsed_time(evs[-1])
    tot = max(_gather(dist, world, mine_ms))
    allr = [m / steps for m in _gather(dist, world, mine_ms)]
    ms = tot / steps
    pts_rank = C5_NXY * C5_NXY * nzl
    res = {"grid_global": [C5_NXY, C5_NXY, nzl * world], "planes_per_rank": nzl,
           "transport": (transport if world > 1 else "none (single GPU)"),
           "steps": steps, "ms_per_step": ms, "gstencils": pts_rank * world / (ms * 1e-3) / 1e9,
           "gstencils_per_gpu": pts_rank / (ms * 1e-3) / 1e9,
           "per_rank_ms_per_step": allr,
           "per_rank_roofline": [{"achieved_GBs": 16 * pts_rank / (m * 1e-3) / 1e9,
                                  "frac": 16 * pts_rank / (m * 1e-3) / 1e9 / peak} for m in allr],
           "rank0_step_ms": {"median": statistics.median(per), "max": max(per)},
           "launches_per_step": launches / steps, "setting_source": s_src,
           "halo_bytes_per_side_per_step": (R * g.pitch_x * g.pitch_y * 8 if world > 1 else 0)}
    if d is not None:
        C.cst_dist_destroy(d)
    del u, v, bufs
    C.cst_stencil_destroy(h)
    torch.cuda.empty_cache()
    return res


def c5_population_eval(C, torch, dist, rank, world, local, n_cand=32, reps=5):
    """configs[4]'s GA part: one GA generation (2 x 16 candidates)
    of star25 settings on the 256 x 1024 x 1024 slab, replayed from a fixed seeded list,
    spread round-robin over the ranks (the cst_dist_tune protocol): each rank times its
    share (2 warm-ups + median of `reps`), then the fitness vectors are all-gathered.  Code
    generation is done before the timed region (warm cubin cache).  evaluations/s = n_cand /
    max-over-ranks wall time of the round (host wall clock: every evaluation synchronises)."""
    import random
    g = C.make_grid(C5_NXY, C5_NXY, C5_WEAK_NZ, R)
    h = C.cst_stencil_create(C.CST_STAR, R, star_coeffs(), g, local)
    count = C.cst_space_count(h)
    rng = random.Random(12345)
    cands = []
    while len(cands) < n_cand:        # the same list on every rank; skip R13 rejections
        s = C.cst_space_at(h, rng.randrange(count))
        if s.as_dict()["bt"] == 1:
            cands.append(s)
    u, v = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(2)]
    C.cst_fill_uniform(g, u.data_ptr(), C5_SEED, 0, C5_NXY, C5_NXY, rank * C5_WEAK_NZ)
    mine = [i for i in range(n_cand) if i % world == rank]
    for i in mine:
        try:
            C.cst_variant_compile(h, cands[i])
        except C.CstError:
            pass
    stream = torch.cuda.current_stream().cuda_stream
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    ms = {}
    for i in mine:
        try:
            ms[i] = C.cst_time_setting(h, cands[i], [u.data_ptr()], [v.data_ptr()], 2, reps,
                                       stream)
        except C.CstError:
            ms[i] = float("inf")
    if world > 1:
        parts = [None] * world
        dist.all_gather_object(parts, ms)
        for p in parts:
            ms.update(p)
    el = max(_gather(dist, world, time.perf_counter() - t0))
    valid = [m for m in ms.values() if m < float("inf")]
    del u, v
    C.cst_stencil_destroy(h)
    torch.cuda.empty_cache()
    return {"candidates": n_cand, "evaluated_by_rank": [len([i for i in range(n_cand)
                                                            if i % world == k])
                                                       for k in range(world)],
            "valid": len(valid), "wall_s_max_over_ranks": el,
            "evaluations_per_s": n_cand / el, "reps_per_eval": reps, "warmup_per_eval": 2,
            "best_ms": min(valid) if valid else None,
            "clock": "host wall clock around the round (evaluations synchronise per candidate)"}


def run_multi(args, C, torch, dist, rank, world, local, shared=False):
    """N > 1: BASELINE configs[4] (see the module docstring).  shared (CST_BENCH_SHARED_GPU,
    tests only): all ranks on one GPU, where NCCL cannot run — the NCCL lines become p2p."""
    peak, peak_src = measured_peaks()
    main_t = "p2p" if shared else "nccl"
    clocks = ClockSampler(local)
    clocks.start()
    weak = c5_sweep(C, torch, dist, rank, world, local, C5_WEAK_NZ, main_t, args.steps,
                    args.warmup, peak)
    clk = clocks.stop()
    strong = c5_sweep(C, torch, dist, rank, world, local, C5_STRONG_NZ // world, main_t,
                      max(3, args.steps // 2), args.warmup, peak)
    p2p = c5_sweep(C, torch, dist, rank, world, local, C5_WEAK_NZ, "p2p", args.steps,
                   args.warmup, peak)
    pop = c5_population_eval(C, torch, dist, rank, world, local)
    if rank == 0:
        pts_rank = C5_NXY * C5_NXY * C5_WEAK_NZ
        r0 = weak["per_rank_roofline"][0]
        line = {"metric": METRIC, "value": weak["gstencils"], "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": max(args.warmup, 3),
                "ms_per_step": weak["ms_per_step"], "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic (cstgen splitmix64 U[-1,1), seed 5, global coordinates per "
                        "slab, device generator)",
                "config": {"workload": "configs[4]: order-4 25-point star (FD Laplacian /5040) "
                                       "z-slab decomposed, 256 x 1024 x 1024 per rank (global "
                                       f"{256 * world} x 1024 x 1024), NCCL halo exchange "
                                       "overlapped with the interior",
                           "grid": weak["grid_global"], "halo": R,
                           "parallelism": f"z-slab x{world}",
                           "l2": "inputs larger than L2 (2 x 2.3 GB per GPU), no flush"},
                "roofline": {"bound": "hbm", "achieved": r0["achieved_GBs"], "peak": peak,
                             "unit": "GB/s", "frac": r0["frac"], "traffic": None,
                             "peak_source": peak_src,
                             "alg_bytes_per_launch": 16 * pts_rank,
                             "kernel": "cst_kernel (star25 slab sweep, rank 0; per-rank "
                                       "fractions under weak.per_rank_roofline)"},
                "clocks": clk, "e2e": None, "cpu_baseline": None,
                "gpu_launches": int(weak["launches_per_step"] * args.steps),
                "weak": weak, "strong": strong, "p2p": p2p, "population_eval": pop,
                "nccl_debug": os.environ.get("NCCL_DEBUG", ""),
                "shared_gpu_test_mode": shared}
        print(json.dumps(line), flush=True)
    dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="cst", choices=["cst", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-other-configs", action="store_true")
    ap.add_argument("--sustained-s", type=float, default=1.5,
                    help="seconds of extra sweeps after the timed region for the steady-state "
                         "(power-capped) line; 0 = skip")
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import torch
    import torch.distributed as dist

    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C

    shared = os.environ.get("CST_BENCH_SHARED_GPU") == "1"
    if shared:   # plumbing test on a one-GPU box: every rank on cuda:0, gloo, p2p only
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            os.environ.setdefault("NCCL_DEBUG", "INFO")        # communicator logs on stderr
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        return run_multi(args, C, torch, dist, rank, world, local, shared)

    # FP64 roofline denominator first, on a cold GPU (boost clock, like the burst-regime
    # timings it divides; measured after minutes of sweeps it reads lower: power cap)
    try:
        fp64_peak, _ = C.cst_fp64_peak(local)
    except Exception:
        fp64_peak = None
    grid = C.make_grid(N, N, N, R)
    h = C.cst_stencil_create(C.CST_STAR, R, star_coeffs(), grid, local)
    s, s_src = load_setting(C, h)
    u = torch.empty(grid.numel, dtype=torch.float64, device="cuda")
    v = torch.empty(grid.numel, dtype=torch.float64, device="cuda")
    stream = torch.cuda.current_stream()
    C.cst_fill_uniform(grid, u.data_ptr(), SEED, 0, N, N, 0, float("nan"), stream.cuda_stream)
    C.cst_fill_uniform(grid, v.data_ptr(), SEED, 0, N, N, 0, float("nan"), stream.cuda_stream)

    def step():
        C.cst_sweep(h, s, [u.data_ptr()], [v.data_ptr()], 1, stream.cuda_stream)

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()
    clocks = ClockSampler(local)
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    torch.cuda.synchronize()
    launches = 0
    clocks.start()
    evs[0].record(stream)
    for i in range(args.steps):
        step()
        launches += C.cst_last_launch_count(h)
        evs[i + 1].record(stream)
    torch.cuda.synchronize()
    clk = clocks.stop()
    per = [evs[i].elapsed_time(evs[i + 1]) for i in range(args.steps)]
    total_ms = evs[0].elapsed_time(evs[-1])
    ms_step = total_ms / args.steps
    pts = N * N * N
    value = pts / (ms_step * 1e-3) / 1e9

    peak, peak_src = measured_peaks()
    avg_launch_ms = statistics.mean(per)
    alg_bytes = 16 * pts                           # read u once + write out once (FP64)
    achieved = alg_bytes / (avg_launch_ms * 1e-3) / 1e9
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": ncu_traffic(), "peak_source": peak_src,
            "alg_bytes_per_launch": alg_bytes, "kernel": "cst_kernel (star25 sweep)",
            "avg_launch_ms": avg_launch_ms, "frac_of_nominal_8TBs": achieved / 8000.0}
    if fp64_peak:
        roof["fp64"] = dict(fp64_from_counters("star25", pts, avg_launch_ms, fp64_peak),
                            fp64_peak_TFLOPs=fp64_peak, fp64_peak_source=FP64_PEAK_SOURCE)

    # ---- steady state: after the timed region, keep sweeping for ~1.5 s and time the
    # launches after the first 0.5 s — the board's 1000 W power cap has then lowered the SM
    # clock (burst vs power-capped regimes); reported beside the headline
    sustained = None
    if args.sustained_s > 0:
        cs = ClockSampler(local)
        cs.start()
        blk, times, t_el = 50, [], 0.0
        while t_el < args.sustained_s * 1e3:
            ev2 = [torch.cuda.Event(enable_timing=True) for _ in range(blk + 1)]
            ev2[0].record(stream)
            for i in range(blk):
                step()
                ev2[i + 1].record(stream)
            torch.cuda.synchronize()
            b = [ev2[i].elapsed_time(ev2[i + 1]) for i in range(blk)]
            times += b
            t_el += sum(b)
        ck = cs.stop()
        cum, steady = 0.0, []
        for m in times:
            cum += m
            if cum >= args.sustained_s * 1e3 / 3:
                steady.append(m)
        sm = statistics.mean(steady)
        sustained = {"ms_per_step": sm, "value": pts / (sm * 1e-3) / 1e9, "unit": UNIT,
                     "hbm_frac": alg_bytes / (sm * 1e-3) / 1e9 / peak, "launches": len(times),
                     "window": f"launches after the first {args.sustained_s / 3:.2f} s of "
                               f"{args.sustained_s:.1f} s of back-to-back sweeps",
                     "clocks": ck}

    # ---- e2e: the same metric through cst_sweep_host (pinned host buffers, H2D + D2H)
    e2e = None
    if args.e2e_steps > 0:
        hu = torch.empty(grid.numel, dtype=torch.float64).pin_memory()
        hv = torch.empty(grid.numel, dtype=torch.float64).pin_memory()
        hu.copy_(u.cpu())
        C.cst_sweep_host(h, s, [hu.data_ptr()], [hv.data_ptr()], 1)     # warm-up / alloc
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            C.cst_sweep_host(h, s, [hu.data_ptr()], [hv.data_ptr()], 1)
        el = (time.perf_counter() - t0) / args.e2e_steps
        # cst_sweep_host uploads every padded plane and row but, per row, only the columns a
        # kernel can read (interior + even x-halo), and reads back the interior
        xh = min(grid.lead_x, grid.halo + (grid.halo & 1))
        xw = min(grid.pitch_x - (grid.lead_x - xh), grid.nx + 2 * xh)
        h2d = (grid.nz + 2 * grid.halo) * grid.pitch_y * xw * 8
        e2e = {"value": pts / el / 1e9, "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": pts * 8, "ms_per_step": el * 1e3,
               "steps": args.e2e_steps, "api": "cst_sweep_host"}

    others = None
    if not args.no_other_configs:
        del u, v
        torch.cuda.empty_cache()
        others = other_configs(C, torch, peak, fp64_peak=fp64_peak)
        others["fp64_peak_TFLOPs_measured"] = fp64_peak
        others["next2_tblock_star7_512_T8"] = tblock_config(C, torch, peak)
        # configs[4] single-GPU baselines (the N = 1 points of the scaling curves)
        others["c5_weak_slab_1gpu"] = c5_sweep(C, torch, None, 0, 1, local, C5_WEAK_NZ, "none",
                                               20, 3, peak)
        others["c5_strong_1gpu"] = c5_sweep(C, torch, None, 0, 1, local, C5_STRONG_NZ, "none",
                                            5, 3, peak)
        others["c5c_population_eval_g1"] = c5_population_eval(C, torch, None, 0, 1, local)

    cpu = None
    if not args.no_cpu_baseline:
        cpu = cpu_baseline()

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": ms_step,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic (cstgen splitmix64 U[-1,1), seed 2, device generator)",
                "config": {"workload": "star25: order-4 25-point star (FD Laplacian /5040), "
                                       "512^3 FP64 interior (BASELINE configs[1])",
                           "grid": [N, N, N], "halo": R,
                           "setting": s.as_dict(), "setting_source": s_src,
                           "l2": "inputs larger than L2 (2 x %.2f GB per GPU), no flush"
                                 % (grid.numel * 8 / 1e9),
                           "parallelism": "single GPU"},
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": clk,
                "sustained": sustained,
                "other_configs": others,
                "gpu_launches": launches,
                "per_step_ms": {"min": min(per), "median": statistics.median(per), "max": max(per),
                                "p90": sorted(per)[int(0.9 * (len(per) - 1))],
                                "slow_steps_gt_1.1x_median":
                                    sum(1 for x in per if x > 1.1 * statistics.median(per))}}
        print(json.dumps(line), flush=True)
    C.cst_stencil_destroy(h)


if __name__ == "__main__":
    main()
