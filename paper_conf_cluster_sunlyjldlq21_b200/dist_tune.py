"""Population-parallel cst_tune over torch.distributed ranks.

The protocol lives in libcst (`cst_dist_tune`, csrc/dist/dist_tune.cpp): rank 0 runs the
tuner, every batch of candidates is broadcast, rank k evaluates candidates i with
i % world == k on its own GPU, and the fitness vectors are all-gathered.  This module only
supplies the host collectives (torch.distributed object collectives, so gloo and NCCL
process groups both work) and argument marshalling.  On a NCCL-transport cst_dist the
library can use its own NCCL communicator instead: call C.cst_dist_tune on that handle.
"""
from __future__ import annotations

import torch.distributed as dist

from . import cst as C


def _collectives(group):
    def bcast(data: bytes, root: int) -> bytes:
        obj = [data]
        dist.broadcast_object_list(obj, src=root, group=group)
        return obj[0]

    def allgather(data: bytes) -> bytes:
        parts = [None] * dist.get_world_size(group)
        dist.all_gather_object(parts, data, group=group)
        return b"".join(parts)
    return bcast, allgather


def tune_distributed(h, opts, in_ptrs, out_ptrs, evaluate_local=None, group=None):
    """Collective over `group`.  evaluate_local(setting_dict) -> ms (or (ms, metrics) when
    opts.n_user_metrics > 0) runs on every rank for its share of each batch; None = libcst's
    built-in GPU timing on in_ptrs / out_ptrs (this rank's replica of the grid).
    Returns (best cst_setting, cst_tune_report) on every rank (rank 0's result)."""
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    bcast, allgather = _collectives(group)
    d, keep = C.cst_dist_create_host(h, world, rank, bcast, allgather)
    local = None
    if evaluate_local is not None:
        nm = opts.n_user_metrics

        def local(settings):
            res = [evaluate_local(s.as_dict()) for s in settings]
            if nm > 0:
                return [r[0] for r in res], [r[1] for r in res]
            return res
    try:
        return C.cst_dist_tune(d, opts, in_ptrs, out_ptrs, local)
    finally:
        C.cst_dist_destroy(d)
        del keep


def gpu_evaluator(stencil, ins, outs, warmup=2, reps=5):
    """evaluate_local for real GPUs: median CUDA-event time of one sweep (Q20)."""
    def ev(d):
        s = C.cst_setting.from_dict(d)
        try:
            return stencil.time_setting(s, ins, outs, warmup=warmup, reps=reps)
        except C.CstError:
            return float("inf")
    return ev
