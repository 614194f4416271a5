"""Run cst_tune (the csTuner pipeline in libcst) on one GPU for a config and record the
tuned setting (used by bench.py) plus the tuner's stage-by-stage JSON report.

    python tools/tune.py --config star25      # BASELINE configs[1]: order-4 star, 512^3
    python tools/tune.py --config box27       # configs[2]
    python tools/tune.py --config hypterm     # configs[3]
    python tools/tune.py --config star25 --start tuned/star25_512.json --refine-all
                                              # hill climb from a recorded setting
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402

D2_R4 = [-9, 128, -1008, 8064, -14350, 8064, -1008, 128, -9]


SIZE_FIELDS = {"tb_x", "tb_y", "tb_z", "sb", "uf_x", "uf_y", "uf_z", "cm_x", "cm_y", "cm_z",
               "bm_x", "bm_y", "bm_z", "bt"}


def neighbours(cur, fixed=(), full=False):
    """Settings one step away from `cur`: SB x2 / /2 and prefetch +-1, or (full) every field
    not in `fixed` (sizes x2 / /2, enumerated fields +-1). Validity is left to
    cst_setting_check; only values below a field's minimum are dropped here."""
    moves = [("sb", (cur["sb"] // 2, cur["sb"] * 2)),
             ("prefetch", (cur["prefetch"] - 1, cur["prefetch"] + 1))]
    if full:
        moves = [(f, (v // 2, v * 2) if f in SIZE_FIELDS else (v - 1, v + 1))
                 for f, v in cur.items() if f not in fixed]
    out = []
    for f, vals in moves:
        for v in vals:
            if v != cur[f] and (v >= 1 or (f not in SIZE_FIELDS and v >= 0)):
                out.append(dict(cur, **{f: v}))
    return out


def config(name):
    if name == "star25":
        w = [v / 5040.0 for v in D2_R4]
        side = w[:4] + w[5:]
        return C.CST_STAR, 4, [3 * w[4]] + side * 3, (512, 512, 512), 2
    if name == "box27":
        b = [0.25, 0.5, 0.25]
        return C.CST_BOX, 1, [x * y * z for x in b for y in b for z in b], (512, 512, 512), 3
    if name == "hypterm":
        return C.CST_HYPTERM, 4, [4 / 5, -1 / 5, 4 / 105, -1 / 280, 1.0, 1.0, 1.0], (512, 512, 512), 4
    if name == "rhs4":
        return C.CST_RHS4, 2, [1.0, 1.0, 1.0], (320, 320, 320), 6
    raise ValueError(name)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="star25")
    ap.add_argument("--budget", type=float, default=300.0)
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=None)
    ap.add_argument("--refine", action="store_true",
                    help="after cst_tune: hill-climb the winner over its SB and prefetch "
                         "neighbours, re-timed (ours, not the paper's; reported separately)")
    ap.add_argument("--refine-all", action="store_true",
                    help="with --refine: the neighbourhood is every field one step away "
                         "(x2 / /2 for sizes, +-1 for enumerated fields), not only SB/prefetch")
    ap.add_argument("--start", default=None,
                    help="tuned JSON to refine from: skips cst_tune and hill-climbs from its "
                         "setting (implies --refine)")
    ap.add_argument("--no-warm-start", action="store_true",
                    help="do not add cst_setting_default() to the dataset (cst_tune_opts."
                         "warm_start = 0): the paper's pipeline from seeded samples only")
    ap.add_argument("--fix", action="append", default=[],
                    help="field=value: tune the sub-space with this field fixed (e.g. "
                         "staging=1); other candidates get fitness 0 through the evaluation "
                         "callback (SURVEY §8(d) C3: each staging mode best-of-tuned)")
    args = ap.parse_args()
    kind, r, coeffs, n, seed = config(args.config)
    g = C.make_grid(*n, r)
    h = C.cst_stencil_create(kind, r, coeffs, g)
    ins = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_IN[kind])]
    outs = [torch.empty(g.numel, dtype=torch.float64, device="cuda") for _ in range(C.N_OUT[kind])]
    for a, t in enumerate(ins):
        C.cst_fill_uniform(g, t.data_ptr(), seed, a)
    torch.cuda.synchronize()
    o = C.cst_tune_opts_default()
    o.seed = args.seed
    o.time_budget_s = args.budget
    o.reps = args.reps
    if args.no_warm_start:
        o.warm_start = 0
    os.makedirs(os.path.join(ROOT, "tuned", "logs"), exist_ok=True)
    tag = "".join(f"_{kv.replace('=', '')}" for kv in args.fix) + ("_nows" if args.no_warm_start else "")
    log = os.path.join(ROOT, "tuned", "logs", f"{args.config}{tag}_seed{args.seed}.json")
    o.log_path = log.encode()
    fixed = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in args.fix}
    eval_fn = None
    if fixed:
        stream0 = torch.cuda.current_stream().cuda_stream

        def eval_fn(settings):
            ms = []
            for st in settings:
                d = st.as_dict()
                if any(d[k] != v for k, v in fixed.items()):
                    ms.append(float("inf"))
                    continue
                try:
                    ms.append(C.cst_time_setting(h, st, [t.data_ptr() for t in ins],
                                                 [t.data_ptr() for t in outs], 2, args.reps,
                                                 stream0))
                except C.CstError:
                    ms.append(float("inf"))
            return ms
        o.warm_start = 0
    t0 = time.time()
    if args.start:
        with open(args.start) as f:
            best = C.cst_setting.from_dict(json.load(f)["setting"])
        rep = None
        args.refine = True
    else:
        best, rep = C.cst_tune(h, o, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs],
                               eval_fn)
    wall = time.time() - t0
    # re-time the winner and the default setting on the same buffers
    stream = torch.cuda.current_stream().cuda_stream
    ms_best = C.cst_time_setting(h, best, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs],
                                 3, 20, stream)
    dflt = C.cst_setting_default(h)
    ms_def = C.cst_time_setting(h, dflt, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs],
                                3, 20, stream)
    refine = None
    if args.refine:
        def timed(st):
            try:
                st = C.cst_setting.from_dict(st) if isinstance(st, dict) else st
                C.cst_setting_check(h, st)
                return C.cst_time_setting(h, st, [t.data_ptr() for t in ins],
                                          [t.data_ptr() for t in outs], 3, 20, stream)
            except (C.CstError, ValueError, OverflowError):
                return float("inf")
        cur, cur_ms, steps = best.as_dict(), ms_best, []
        for _ in range(3):
            cands = neighbours(cur, fixed, args.refine_all)
            timed_c = [(timed(d), d) for d in cands]
            ms_c, d_c = min(timed_c, key=lambda x: x[0])
            steps.append({"from_ms": cur_ms,
                          "neighbours": [[m, {k: v for k, v in d.items() if cur[k] != v}]
                                         for m, d in timed_c]})
            if ms_c < 0.99 * cur_ms:
                cur, cur_ms = d_c, ms_c
            else:
                break
        refine = {"tuned_setting": best.as_dict(), "tuned_retimed_ms": ms_best, "steps": steps}
        best, ms_best = C.cst_setting.from_dict(cur), cur_ms
    pts = n[0] * n[1] * n[2]
    res = {"config": args.config, "grid": list(n), "setting": best.as_dict(),
           "tuned_ms": rep.best_ms if rep else None, "retimed_ms": ms_best, "gstencils": pts / (ms_best * 1e-3) / 1e9,
           "default_setting": dflt.as_dict(), "default_ms": ms_def,
           "report": {f: getattr(rep, f) for f, _ in rep._fields_} if rep else None,
           "wall_s": wall, "start": args.start,
           "log": os.path.relpath(log, ROOT), "seed": args.seed, "budget_s": args.budget,
           "fixed": fixed, "refine": refine}
    if args.start:
        tag += "_refined"
    out = args.out or os.path.join(ROOT, "tuned", f"{args.config}_{n[0]}{tag}.json")
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res))
    C.cst_stencil_destroy(h)


if __name__ == "__main__":
    main()
