"""Torch-tensor convenience layer over the C ABI (plumbing only: device memory + streams).

    st = Stencil(CST_STAR, 4, coeffs, make_grid(512, 512, 512, 4))
    u, v = st.empty(2)                       # padded FP64 device grids
    st.fill(u, seed=2, array_id=0)           # cstgen values (device twin)
    s = st.default_setting()
    st.sweep(s, [u], [v])                    # libcst kernels on the current stream
"""
from __future__ import annotations

import torch

from . import cst as C


class Stencil:
    def __init__(self, kind: int, order: int, coeffs, grid: C.cst_grid, device: int = 0):
        self.kind, self.order = kind, order
        self.coeffs = [float(c) for c in coeffs]
        self.grid = grid
        self.device = device
        self.n_in, self.n_out = C.N_IN[kind], C.N_OUT[kind]
        self.h = C.cst_stencil_create(kind, order, self.coeffs, grid, device)

    def close(self):
        if self.h:
            C.cst_stencil_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ------------------------------------------------------------ memory (torch)
    def empty(self, n: int = 1, fill=float("nan")):
        out = []
        for _ in range(n):
            t = torch.empty(self.grid.numel, dtype=torch.float64, device=f"cuda:{self.device}")
            if fill is not None:
                t.fill_(fill)
            out.append(t)
        return out

    def view(self, t: torch.Tensor) -> torch.Tensor:
        """[z][y][x] view of the logical padded region [-h, n+h)^3."""
        g = self.grid
        h = g.halo
        a = t.view(g.nz + 2 * h, g.pitch_y, g.pitch_x)
        return a[:, : g.ny + 2 * h, g.lead_x - h: g.lead_x + g.nx + h]

    def interior(self, t: torch.Tensor) -> torch.Tensor:
        g = self.grid
        h = g.halo
        return self.view(t)[h:h + g.nz, h:h + g.ny, h:h + g.nx]

    def fill(self, t: torch.Tensor, seed: int, array_id: int, nx_global=None, ny_global=None,
             z0: int = 0, pad_value: float = float("nan")):
        C.cst_fill_uniform(self.grid, t.data_ptr(), seed, array_id, nx_global, ny_global, z0,
                           pad_value, torch.cuda.current_stream(self.device).cuda_stream)

    # ------------------------------------------------------------ ABI calls
    def default_setting(self) -> C.cst_setting:
        return C.cst_setting_default(self.h)

    def check(self, s: C.cst_setting) -> None:
        C.cst_setting_check(self.h, s)

    def space_count(self) -> int:
        return C.cst_space_count(self.h)

    def space_at(self, rank: int) -> C.cst_setting:
        return C.cst_space_at(self.h, rank)

    def space_rank(self, s: C.cst_setting) -> int:
        return C.cst_space_rank(self.h, s)

    def kernel_info(self, s: C.cst_setting) -> C.cst_kernel_info:
        return C.cst_kernel_info_get(self.h, s)

    def sweep(self, s: C.cst_setting, ins, outs, nsteps: int = 1, stream=None) -> None:
        st = stream if stream is not None else torch.cuda.current_stream(self.device)
        C.cst_sweep(self.h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs], nsteps,
                    st.cuda_stream)

    def sweep_host(self, s: C.cst_setting, ins, outs, nsteps: int = 1) -> None:
        C.cst_sweep_host(self.h, s, [t.data_ptr() for t in ins], [t.data_ptr() for t in outs],
                         nsteps)

    def time_setting(self, s, ins, outs, warmup=2, reps=5, stream=None) -> float:
        st = stream if stream is not None else torch.cuda.current_stream(self.device)
        return C.cst_time_setting(self.h, s, [t.data_ptr() for t in ins],
                                  [t.data_ptr() for t in outs], warmup, reps, st.cuda_stream)

    def last_launch_count(self) -> int:
        return C.cst_last_launch_count(self.h)

    def sync(self) -> None:
        C.cst_sync(self.h)
