"""Multi-process (gloo, world_size 2, CPU) tests of the N>1 host logic.

1. z-slab decomposition: each rank sweeps its slab with the oracle and exchanges halo
   planes per libcst's cst_dist_halo_plan through torch.distributed send/recv; after T
   steps the slabs reassemble BIT-IDENTICALLY into the global T-step oracle result.
2. population-parallel tuning: cst_tune on rank 0 with every batch spread over both
   ranks gives exactly the single-process result (same seed -> same trajectory).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import cstgen
from oracle import stencil as ost


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world,
                            init_method=f"tcp://127.0.0.1:{port}")


# ------------------------------------------------------------------ 1. z-slab exchange
NX, NY, NZL, R, T, SEED = 12, 10, 6, 2, 3, 17


def _slab_worker(rank, world, port, outdir):
    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
    _init(rank, world, port)
    c = ost.star_laplacian_coeffs(R)
    L = cstgen.make_layout(NX, NY, NZL, R)
    z0 = rank * NZL
    a = cstgen.fill(L, SEED, 0, z0=z0)       # true neighbour values in the halos at t=0
    b = a.copy()
    plane = L.pitch_y * L.pitch_x
    plan = C.cst_dist_halo_plan(world, rank, NZL, R)
    src, dst = a, b
    for _ in range(T):
        ost.sweep(1, R, c, L, [src], [dst], nsteps=1)
        reqs = []
        for peer, is_send, p0, n in plan:
            off = (p0 + L.halo) * plane
            view = torch.from_numpy(dst[off:off + n * plane])
            if is_send:
                reqs.append(dist.isend(view.clone(), dst=peer))
            else:
                buf = torch.empty(n * plane, dtype=torch.float64)
                reqs.append((dist.irecv(buf, src=peer), view, buf))
        for q in reqs:
            if isinstance(q, tuple):
                q[0].wait()
                q[1].copy_(q[2])
            else:
                q.wait()
        src, dst = dst, src
    np.save(os.path.join(outdir, f"slab{rank}.npy"), src)
    dist.barrier()
    dist.destroy_process_group()


def test_zslab_exchange_matches_global_oracle(tmp_path):
    world = 2
    mp.spawn(_slab_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    c = ost.star_laplacian_coeffs(R)
    G = cstgen.make_layout(NX, NY, NZL * world, R)
    a = cstgen.fill(G, SEED, 0)
    b = a.copy()
    ost.sweep(1, R, c, G, [a], [b], nsteps=T)
    res = b if T % 2 else a
    gv = G.view(res)
    L = cstgen.make_layout(NX, NY, NZL, R)
    for rank in range(world):
        s = L.view(np.load(tmp_path / f"slab{rank}.npy"))
        z0 = rank * NZL
        got = s[R:R + NZL]
        want = gv[R + z0:R + z0 + NZL]
        assert np.array_equal(got, want), rank


def test_halo_plan_shapes():
    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
    assert C.cst_dist_halo_plan(1, 0, 8, 4) == []
    assert C.cst_dist_halo_plan(4, 0, 8, 4) == [(1, 1, 4, 4), (1, 0, 8, 4)]
    assert C.cst_dist_halo_plan(4, 3, 8, 4) == [(2, 1, 0, 4), (2, 0, -4, 4)]
    with pytest.raises(C.CstError):
        C.cst_dist_halo_plan(2, 0, 7, 4)          # nz < 2r


# ------------------------------------------------------------------ 2. population-parallel GA
def _tune_worker(rank, world, port, outdir):
    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
    from paper_conf_cluster_sunlyjldlq21_b200.dist_tune import tune_distributed
    import test_tuner as TT
    _init(rank, world, port)
    g = C.make_grid(*TT.M, TT.R)
    h = C.cst_stencil_create(TT.KIND, TT.R, [1.0] * 7, g)
    o = C.cst_tune_opts_default()
    o.seed = 9
    o.n_user_metrics = TT.NMET
    o.time_budget_s = 0
    o.warm_start = 0
    evaluated = []

    def ev(d):
        evaluated.append(tuple(d[f] for f in C.FIELDS))
        return TT.synth(d)

    best, rep = tune_distributed(h, o, [], [], ev)
    np.save(os.path.join(outdir, f"tune{rank}.npy"),
            np.array(list(best.as_tuple()) + [len(evaluated)], dtype=np.int64))
    if rank == 0:
        np.save(os.path.join(outdir, "rep.npy"), np.array([rep.best_ms, rep.evaluations]))
    C.cst_stencil_destroy(h)
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_population_parallel_tuning_equals_single_process(tmp_path, world):
    """Same seed -> the same result and report for 1, 2 and 4 evaluating ranks (SURVEY
    8(c) GA pin: the trajectory does not depend on the number of evaluators)."""
    import test_tuner as TT
    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
    mp.spawn(_tune_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    rs = [np.load(tmp_path / f"tune{k}.npy") for k in range(world)]
    r0 = rs[0]
    for r in rs[1:]:
        assert np.array_equal(r0[:-1], r[:-1])              # every rank knows the best setting
    assert all(r[-1] > 0 for r in rs)                         # every rank evaluated candidates
    g = C.make_grid(*TT.M, TT.R)
    h = C.cst_stencil_create(TT.KIND, TT.R, [1.0] * 7, g)
    o = C.cst_tune_opts_default()
    o.seed = 9
    o.n_user_metrics = TT.NMET
    o.time_budget_s = 0
    o.warm_start = 0
    best, rep = C.cst_tune(h, o, [], [], eval_fn=lambda ss: (
        [TT.synth(s.as_dict())[0] for s in ss], [TT.synth(s.as_dict())[1] for s in ss]))
    C.cst_stencil_destroy(h)
    assert tuple(r0[:-1]) == best.as_tuple()
    rep_d = np.load(tmp_path / "rep.npy")
    assert rep_d[0] == rep.best_ms and int(rep_d[1]) == rep.evaluations


def _tune_fail_worker(rank, world, port, outdir):
    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
    from paper_conf_cluster_sunlyjldlq21_b200.dist_tune import tune_distributed
    import test_tuner as TT
    _init(rank, world, port)
    g = C.make_grid(*TT.M, TT.R)
    h = C.cst_stencil_create(TT.KIND, TT.R, [1.0] * 7, g)
    o = C.cst_tune_opts_default()
    o.n_user_metrics = TT.NMET
    o.time_budget_s = 0

    def ev(d):                     # every candidate fails -> rank 0's tuner fails
        raise RuntimeError("evaluation failed")

    status = "ok"
    try:
        tune_distributed(h, o, [], [], ev)
    except C.CstError as e:
        status = f"{e.status}"
    with open(os.path.join(outdir, f"fail{rank}.txt"), "w") as f:
        f.write(status)
    C.cst_stencil_destroy(h)
    dist.destroy_process_group()


def test_population_parallel_tuning_error_reaches_every_rank(tmp_path):
    """if rank 0's tuner fails, the result message is still broadcast, so every
    rank returns the error instead of blocking."""
    world = 2
    mp.spawn(_tune_fail_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world,
             join=True)
    got = [open(tmp_path / f"fail{k}.txt").read() for k in range(world)]
    assert got[0] == got[1] != "ok", got

