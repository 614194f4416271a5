"""bench.py — GStencil/s of the complex-stencil sweep on B200 (BASELINE.json configs[1]).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl cst|reference]

N=1 workload: order-4 25-point star (FD Laplacian, weights /5040), 512^3 FP64 interior,
halo 4, the tuned setting from tuned/star25_512.json (cst_tune output, then the A/B-checked
hill climb of tools/tune.py --refine-all; the default setting if absent).  A step = one sweep (one kernel launch) over inputs resident in HBM; the two
1.18 GB arrays exceed the 126 MB L2, so no flush is needed between steps.
N>1 (torchrun, one rank per GPU): weak scaling of the z-slab decomposition — every rank owns
a 512^3 slab of a (512*N) x 512 x 512 grid and exchanges 4-plane halos with its neighbours
every step (cst_dist_sweep: by default the boundary kernels store straight into the
neighbours' halos over peer memory, --halo nccl selects NCCL send/recv overlapped with the
interior).  value = all ranks' points / max-over-ranks time.

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


def other_configs(C, torch, peak, steps=10, fp64_peak=None):
    """The other single-GPU configs of BASELINE.json, each timed the same way (CUDA events,
    inputs resident, device generator), with their own roofline fractions."""
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
        ms = C.cst_time_setting(h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs],
                                3, steps, torch.cuda.current_stream().cuda_stream)
        pts = n[0] * n[1] * n[2]
        bpp = 8 * (C.N_IN[kind] + C.N_OUT[kind])
        gbs = pts * bpp / (ms * 1e-3) / 1e9
        res[name] = {"workload": desc, "gstencils": pts / (ms * 1e-3) / 1e9, "ms_median": ms,
                     "alg_bytes_per_point": bpp, "achieved_GBs": gbs,
                     "hbm_frac_measured": None if n[0] < 128 else gbs / peak,
                     "hbm_frac_nominal_8TBs": None if n[0] < 128 else gbs / 8000.0,
                     "setting": s.as_dict(), "setting_source": src}
        fpp = FLOPS_PER_POINT.get(kind)
        if fpp and fp64_peak:
            tf = pts * fpp / (ms * 1e-3) / 1e12
            res[name].update({"flops_per_point_as_written": fpp, "achieved_TFLOPs": tf,
                              "fp64_frac_measured": tf / fp64_peak})
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="cst", choices=["cst", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-other-configs", action="store_true")
    ap.add_argument("--halo", default=os.environ.get("CST_BENCH_HALO", "p2p"),
                    choices=["p2p", "nccl"],
                    help="N > 1: fused peer-memory halo stores (default) or NCCL send/recv")
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import torch
    import torch.distributed as dist

    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    grid = C.make_grid(N, N, N, R)
    h = C.cst_stencil_create(C.CST_STAR, R, star_coeffs(), grid, local)
    s, s_src = load_setting(C, h)
    u = torch.empty(grid.numel, dtype=torch.float64, device="cuda")
    v = torch.empty(grid.numel, dtype=torch.float64, device="cuda")
    stream = torch.cuda.current_stream()
    z0 = rank * N
    C.cst_fill_uniform(grid, u.data_ptr(), SEED, 0, N, N, z0, float("nan"), stream.cuda_stream)
    C.cst_fill_uniform(grid, v.data_ptr(), SEED, 0, N, N, z0, float("nan"), stream.cuda_stream)
    dist_h = None
    halo_used = args.halo
    if world > 1 and args.halo == "p2p":
        # boundary kernels store straight into the neighbours' halos (NVLink peer stores).
        # Every rank must take the same transport: export, all-gather (ok, blob), import,
        # agree by MIN-reduce; any failure anywhere -> all ranks fall back to NCCL.
        dist_h = C.cst_dist_create(h, world, rank, None)
        ok, why, mine = True, "", None
        try:
            mine = C.cst_dist_p2p_export(dist_h, [u.data_ptr()], [v.data_ptr()])
        except C.CstError as e:
            ok, why = False, str(e)
        blobs = [None] * world
        dist.all_gather_object(blobs, (ok, mine))
        if ok and all(b[0] for b in blobs):
            try:
                for peer in (rank - 1, rank + 1):
                    if 0 <= peer < world:
                        C.cst_dist_p2p_import(dist_h, peer, blobs[peer][1])
            except C.CstError as e:
                ok, why = False, str(e)
        else:
            ok, why = False, why or "a peer could not export"
        flag = torch.tensor([1 if ok else 0], device="cuda")
        dist.all_reduce(flag, op=dist.ReduceOp.MIN)
        if int(flag.item()) == 0:
            C.cst_dist_destroy(dist_h)
            dist_h = None
            halo_used = "nccl (p2p setup failed: %s)" % (why or "on another rank")[:120]
    if world > 1 and dist_h is None:
        uid = C.cst_dist_nccl_unique_id() if rank == 0 else None
        obj = [uid]
        dist.broadcast_object_list(obj, src=0)
        dist_h = C.cst_dist_create(h, world, rank, obj[0])

    def step():
        if dist_h is not None:
            C.cst_dist_sweep(dist_h, s, [u.data_ptr()], [v.data_ptr()], 1, stream.cuda_stream)
        else:
            C.cst_sweep(h, s, [u.data_ptr()], [v.data_ptr()], 1, stream.cuda_stream)

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = ClockSampler(local)
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = 0
    clocks.start()
    evs[0].record(stream)
    for i in range(args.steps):
        step()
        launches += C.cst_last_launch_count(h)
        evs[i + 1].record(stream)
    torch.cuda.synchronize()
    clk = clocks.stop()
    if world > 1:
        dist.barrier()
    per = [evs[i].elapsed_time(evs[i + 1]) for i in range(args.steps)]
    total_ms = evs[0].elapsed_time(evs[-1])
    if world > 1:
        t = torch.tensor([total_ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_step = total_ms / args.steps
    pts = N * N * N
    value = pts * world / (ms_step * 1e-3) / 1e9

    peak, peak_src = measured_peaks()
    avg_launch_ms = statistics.mean(per)
    alg_bytes = 16 * pts                           # read u once + write out once (FP64)
    achieved = alg_bytes / (avg_launch_ms * 1e-3) / 1e9
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": ncu_traffic(), "peak_source": peak_src,
            "alg_bytes_per_launch": alg_bytes, "kernel": "cst_kernel (star25 sweep)",
            "avg_launch_ms": avg_launch_ms, "frac_of_nominal_8TBs": achieved / 8000.0}

    # ---- e2e: the same metric through cst_sweep_host (pinned host buffers, H2D + D2H)
    e2e = None
    if rank == 0 and world == 1 and args.e2e_steps > 0:
        hu = torch.empty(grid.numel, dtype=torch.float64).pin_memory()
        hv = torch.empty(grid.numel, dtype=torch.float64).pin_memory()
        hu.copy_(u.cpu())
        C.cst_sweep_host(h, s, [hu.data_ptr()], [hv.data_ptr()], 1)     # warm-up / alloc
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            C.cst_sweep_host(h, s, [hu.data_ptr()], [hv.data_ptr()], 1)
        el = (time.perf_counter() - t0) / args.e2e_steps
        e2e = {"value": pts / el / 1e9, "unit": UNIT, "h2d_bytes_per_step": grid.numel * 8,
               "d2h_bytes_per_step": pts * 8, "ms_per_step": el * 1e3,
               "steps": args.e2e_steps, "api": "cst_sweep_host"}

    others = None
    if rank == 0 and world == 1 and not args.no_other_configs:
        del u, v
        torch.cuda.empty_cache()
        try:
            fp64_peak, _ = C.cst_fp64_peak(local)
        except Exception:
            fp64_peak = None
        others = other_configs(C, torch, peak, fp64_peak=fp64_peak)
        others["fp64_peak_TFLOPs_measured"] = fp64_peak
        others["next2_tblock_star7_512_T8"] = tblock_config(C, torch, peak)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline()

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": ms_step,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic (cstgen splitmix64 U[-1,1), seed 2, device generator)",
                "config": {"workload": "star25: order-4 25-point star (FD Laplacian /5040), "
                                       "512^3 FP64 interior per GPU (BASELINE configs[1])"
                                       + (("; z-slab weak scaling, halo exchange: "
                                           + ("fused peer-memory stores" if halo_used == "p2p"
                                              else "NCCL send/recv" if halo_used == "nccl"
                                              else halo_used)) if world > 1 else ""),
                           "grid": [N, N, N * world], "halo": R,
                           "setting": s.as_dict(), "setting_source": s_src,
                           "l2": "inputs larger than L2 (2 x %.2f GB per GPU), no flush"
                                 % (grid.numel * 8 / 1e9),
                           "parallelism": f"z-slab x{world}" if world > 1 else "single GPU"},
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": clk,
                "other_configs": others,
                "gpu_launches": launches,
                "per_step_ms": {"min": min(per), "median": statistics.median(per), "max": max(per),
                                "p90": sorted(per)[int(0.9 * (len(per) - 1))],
                                "slow_steps_gt_1.1x_median":
                                    sum(1 for x in per if x > 1.1 * statistics.median(per))}}
        print(json.dumps(line), flush=True)
    if dist_h is not None:
        C.cst_dist_destroy(dist_h)
    C.cst_stencil_destroy(h)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
