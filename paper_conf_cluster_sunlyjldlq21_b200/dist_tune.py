"""Population-parallel evaluation for cst_tune (SURVEY §8(e), P:296 multi-process GA).

Rank 0 runs the C++ tuner; every batch of candidates it asks for (the 128-setting dataset,
then each GA generation of 2 x 16 individuals) is spread round-robin over all ranks, each
rank evaluates its share on its own GPU (libcst: NVRTC code generation + CUDA-event timing)
and the fitness vectors are all-gathered through torch.distributed (host coordination,
8 B per candidate).  The GA itself stays on rank 0 and is deterministic, so the trajectory
does not depend on the number of evaluating ranks.
"""
from __future__ import annotations

import torch.distributed as dist

from . import cst as C

_STOP = "__cst_tune_stop__"


def _share(batch, rank, world):
    return [(i, t) for i, t in enumerate(batch) if i % world == rank]


def _merge(parts, n):
    out = [None] * n
    for part in parts:
        for i, v in part:
            out[i] = v
    return out


def tune_distributed(h, opts, in_ptrs, out_ptrs, evaluate_local, group=None):
    """Collective over `group`.  evaluate_local(setting_dict) -> ms (or (ms, metrics) when
    opts.n_user_metrics > 0) runs on every rank for its share of each batch.
    Returns (best cst_setting, cst_tune_report or None on ranks != 0) on every rank."""
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    nm = opts.n_user_metrics

    def serve(batch):
        mine = [(i, evaluate_local(dict(zip(C.FIELDS, t)))) for i, t in _share(batch, rank, world)]
        parts = [None] * world
        dist.all_gather_object(parts, mine, group=group)
        return _merge(parts, len(batch))

    if rank == 0:
        def cb(settings):
            batch = [s.as_tuple() for s in settings]
            dist.broadcast_object_list([batch], src=0, group=group)
            res = serve(batch)
            if nm > 0:
                return [r[0] for r in res], [r[1] for r in res]
            return res

        try:
            best, rep = C.cst_tune(h, opts, in_ptrs, out_ptrs, eval_fn=cb)
        finally:
            dist.broadcast_object_list([_STOP], src=0, group=group)
        obj = [best.as_dict()]
        dist.broadcast_object_list(obj, src=0, group=group)
        return best, rep
    while True:
        obj = [None]
        dist.broadcast_object_list(obj, src=0, group=group)
        if isinstance(obj[0], str) and obj[0] == _STOP:
            break
        serve(obj[0])
    obj = [None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return C.cst_setting.from_dict(obj[0]), None


def gpu_evaluator(stencil, ins, outs, warmup=2, reps=5):
    """evaluate_local for real GPUs: median CUDA-event time of one sweep (Q20)."""
    def ev(d):
        s = C.cst_setting.from_dict(d)
        try:
            return stencil.time_setting(s, ins, outs, warmup=warmup, reps=reps)
        except C.CstError:
            return float("inf")
    return ev
