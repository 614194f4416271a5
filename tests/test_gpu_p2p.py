"""Fused peer-memory halo exchange: two processes, one z-slab each,
exchange halos only through the boundary kernels' stores into the neighbour's IPC-mapped
buffers and flag words (no NCCL, no copies).  On the one-GPU test box both processes share
cuda:0 (CUDA IPC works between processes on one device; contexts time-slice, so the flag
waits see the peer's progress).  The slabs must reproduce the single-grid sweep bit for bit,
for one and several ping-pong steps, with both buffer orders."""
import os
import tempfile

import numpy as np
import pytest

torch = pytest.importorskip("torch")

from cst_testutil import gpu_available  # noqa: E402

pytestmark = pytest.mark.gpu
if not gpu_available():
    pytest.skip("no GPU", allow_module_level=True)

NX, NY, NZL, SEED = 64, 40, 16, 31
SETTING = dict(tb_x=32, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=8,
               uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=2, bm_y=2, bm_z=1,
               use_retiming=2, prefetch=2, bt=1)


def _coeffs(kind, R):
    import gpu_helpers as H
    return list(H.coeffs(kind, R, "random", seed=5))


def _worker(rank, world, port, out_dir, calls, kind, R, nan_out):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    import torch
    import torch.distributed as dist
    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        ls = C.make_grid(NX, NY, NZL, R)
        h = C.cst_stencil_create(kind, R, _coeffs(kind, R), ls)
        a = torch.empty(ls.numel, dtype=torch.float64, device="cuda")
        b = torch.empty(ls.numel, dtype=torch.float64, device="cuda")
        for t in (a, b):
            C.cst_fill_uniform(ls, t.data_ptr(), SEED, 0, NX, NY, rank * NZL)
        if nan_out:               # out starts as garbage: every halo value it needs must be
            b.fill_(float("nan"))  # copied (x/y ring) or exchanged (interior of z-halo planes)
        d = C.cst_dist_create(h, world, rank, None)
        C.cst_dist_p2p_setup(d, rank, world, [a.data_ptr()], [b.data_ptr()])
        s = C.cst_setting.from_dict(SETTING)
        cur_in, cur_out = a, b
        for nsteps in calls:            # consecutive calls continue the flag epochs
            C.cst_dist_sweep(d, s, [cur_in.data_ptr()], [cur_out.data_ptr()], nsteps)
            if nsteps % 2:
                cur_in, cur_out = cur_out, cur_in
        C.cst_sync(h)
        launches = C.cst_last_launch_count(h)
        np.save(os.path.join(out_dir, f"r{rank}.npy"), cur_in.cpu().numpy())
        np.save(os.path.join(out_dir, f"n{rank}.npy"), np.array([launches]))
        dist.barrier()
        C.cst_dist_destroy(d)
        C.cst_stencil_destroy(h)
    finally:
        dist.destroy_process_group()


def _free_port():
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("kind,R,nan_out", [(1, 4, False), (2, 1, True), (1, 4, True)],
                         ids=["star25", "box27-nan-out", "star25-nan-out"])
@pytest.mark.parametrize("calls", [[1], [3], [2, 1]], ids=["1step", "3steps", "2+1steps"])
def test_p2p_slabs_bit_identical_to_single_grid(calls, kind, R, nan_out):
    import torch.multiprocessing as mp
    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
    world = 2
    total = sum(calls)
    gl = C.make_grid(NX, NY, NZL * world, R)
    hg = C.cst_stencil_create(kind, R, _coeffs(kind, R), gl)
    ug, vg = [torch.empty(gl.numel, dtype=torch.float64, device="cuda") for _ in range(2)]
    for t in (ug, vg):
        C.cst_fill_uniform(gl, t.data_ptr(), SEED, 0)
    if nan_out:
        vg.fill_(float("nan"))
    C.cst_sweep(hg, C.cst_setting.from_dict(SETTING), [ug.data_ptr()], [vg.data_ptr()], total)
    C.cst_sync(hg)
    glob = (vg if total % 2 else ug).cpu().numpy()
    C.cst_stencil_destroy(hg)
    with tempfile.TemporaryDirectory() as td:
        mp.start_processes(_worker, args=(world, _free_port(), td, calls, kind, R, nan_out),
                           nprocs=world,
                           join=True, start_method="spawn")
        ls = C.make_grid(NX, NY, NZL, R)
        plane = ls.pitch_y * ls.pitch_x
        for k in range(world):
            res = np.load(os.path.join(td, f"r{k}.npy"))
            # interior planes and the halo planes received from the neighbours
            lo = 0 if k == 0 else -R
            hi = NZL if k == world - 1 else NZL + R
            mine = res[(R + lo) * plane:(R + hi) * plane]
            ref = glob[(R + k * NZL + lo) * plane:(R + k * NZL + hi) * plane]
            m = np.zeros((hi - lo, ls.pitch_y, ls.pitch_x), bool)
            m[:, R:R + NY, ls.lead_x:ls.lead_x + NX] = True
            got, want = mine.reshape(m.shape)[m], ref.reshape(m.shape)[m]
            assert np.array_equal(got.view(np.uint64), want.view(np.uint64)), f"slab {k}"
            n = int(np.load(os.path.join(td, f"n{k}.npy"))[0])
            assert n == calls[-1] * (3 + 4)       # per step: 3 sweeps + 2 waits + 2 signals
