"""Config 5 (BASELINE configs[4]): order-4 star on a z-slab decomposed grid over N GPUs.

    torchrun --nproc-per-node N --master-addr 127.0.0.1 tools/scaling.py --mode strong
    torchrun --nproc-per-node N --master-addr 127.0.0.1 tools/scaling.py --mode weak

strong: the 2048 x 1024 x 1024 (nz, ny, nx) global grid split into N slabs of 2048/N planes.
weak:   256 x 1024 x 1024 per rank (global nz = 256 N).
T = 10 steps (ping-pong, NCCL halo exchange each step) after 3 warm-up steps; time =
max over ranks of CUDA-event time; prints one JSON line on rank 0.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402

D2_R4 = [-9, 128, -1008, 8064, -14350, 8064, -1008, 128, -9]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--mode", choices=["strong", "weak"], default="weak")
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--setting", default=os.path.join(ROOT, "tuned", "star25_512.json"))
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    nx = ny = 1024
    nzl = 2048 // world if args.mode == "strong" else 256
    r = 4
    w = [v / 5040.0 for v in D2_R4]
    coeffs = [3 * w[4]] + (w[:4] + w[5:]) * 3
    g = C.make_grid(nx, ny, nzl, r)
    h = C.cst_stencil_create(C.CST_STAR, r, coeffs, g, local)
    if os.path.exists(args.setting):
        s = C.cst_setting.from_dict(json.load(open(args.setting))["setting"])
        try:
            C.cst_setting_check(h, s)
        except C.CstError:
            s = C.cst_setting_default(h)
    else:
        s = C.cst_setting_default(h)
    u, v = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(2)]
    for t in (u, v):
        C.cst_fill_uniform(g, t.data_ptr(), 5, 0, nx, ny, rank * nzl)
    uid = C.cst_dist_nccl_unique_id() if rank == 0 else None
    if world > 1:
        obj = [uid]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    d = C.cst_dist_create(h, world, rank, uid)
    stream = torch.cuda.current_stream()
    C.cst_dist_sweep(d, s, [u.data_ptr()], [v.data_ptr()], args.warmup, stream.cuda_stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    C.cst_dist_sweep(d, s, [u.data_ptr()], [v.data_ptr()], args.steps, stream.cuda_stream)
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    pts = nx * ny * nzl * world
    gst = pts * args.steps / (ms * 1e-3) / 1e9
    if rank == 0:
        print(json.dumps({"mode": args.mode, "n_gpus": world, "grid": [nx, ny, nzl * world],
                          "steps": args.steps, "ms_per_step": ms / args.steps, "gstencils": gst,
                          "gstencils_per_gpu": gst / world, "setting": s.as_dict(),
                          "hbm_frac_measured": gst * 16 / world / 6549.4}))
    C.cst_dist_destroy(d)
    C.cst_stencil_destroy(h)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
