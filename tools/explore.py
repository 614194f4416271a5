"""Time a list of hand-picked settings of a config on the GPU (exploration, not the bench)."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402


def base(**kw):
    d = dict(tb_x=64, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=128,
             uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=1, bm_y=1, bm_z=1,
             use_retiming=2, prefetch=3, bt=1)
    d.update(kw)
    return d


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kind", type=int, default=1)
    ap.add_argument("--order", type=int, default=4)
    ap.add_argument("--n", type=int, nargs=3, default=[512, 512, 512])
    ap.add_argument("--settings", default=None, help="json file with a list of setting dicts")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--nsteps", type=int, default=1, help="steps per cst_sweep (ms per step)")
    args = ap.parse_args()
    kind, r = args.kind, args.order
    nc = {1: 6 * r + 1, 2: 27, 3: 7, 4: 3}[kind]
    coeffs = [0.1] * nc
    g = C.make_grid(*args.n, r)
    h = C.cst_stencil_create(kind, r, coeffs, g)
    nin, nout = C.N_IN[kind], C.N_OUT[kind]
    ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(nin)]
    outs = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(nout)]
    for a, t in enumerate(ins):
        C.cst_fill_uniform(g, t.data_ptr(), 1, a)
    torch.cuda.synchronize()
    if args.settings:
        settings = json.load(open(args.settings))
    else:
        settings = [base()]
    pts = args.n[0] * args.n[1] * args.n[2]
    bytes_pt = 8 * (nin + nout)
    res = []
    for d in settings:
        s = C.cst_setting.from_dict(base(**d))
        try:
            info = C.cst_kernel_info_get(h, s)
            ms = C.cst_time_setting(h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs],
                                    2, args.reps, torch.cuda.current_stream().cuda_stream,
                                    nsteps=args.nsteps)
        except C.CstError as e:
            print(json.dumps({"setting": d, "error": str(e)}), flush=True)
            continue
        gst = pts / (ms * 1e-3) / 1e9
        row = {"setting": d, "nsteps": args.nsteps, "ms": round(ms, 4), "gst": round(gst, 1),
               "GBs": round(gst * bytes_pt, 1), "regs": info.registers, "smem": info.smem_bytes,
               "occ": info.ctas_per_sm, "ctas": info.grid_ctas}
        res.append(row)
        print(json.dumps(row), flush=True)
    res.sort(key=lambda x: -x["gst"])
    print("BEST", json.dumps(res[:5]))


if __name__ == "__main__":
    main()
