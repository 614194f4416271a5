"""ctypes wrapper of liboracle.so — the CPU definition of the sweep (oracle/oracle.cpp).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from cstgen import Layout

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

STAR, BOX, HYPTERM, RHS4 = 1, 2, 3, 4
N_IN = {STAR: 1, BOX: 1, HYPTERM: 8, RHS4: 5}
N_OUT = {STAR: 1, BOX: 1, HYPTERM: 5, RHS4: 3}

_DP = ctypes.POINTER(ctypes.c_double)


def build() -> str:
    """Compile liboracle.so (plain g++, no FMA contraction, OpenMP over z)."""
    src = os.path.join(_HERE, "oracle.cpp")
    if (not os.path.exists(_LIB_PATH)) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(
            ["g++", "-std=c++17", "-O3", "-fno-fast-math", "-ffp-contract=off", "-fopenmp",
             "-fPIC", "-shared", "-o", _LIB_PATH, src])
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        i64 = ctypes.c_int64
        L.oracle_sweep.argtypes = [ctypes.c_int, ctypes.c_int, _DP, i64, i64, i64, i64, i64, i64,
                                   i64, ctypes.POINTER(_DP), ctypes.POINTER(_DP), ctypes.c_int,
                                   ctypes.c_int]
        L.oracle_sweep.restype = ctypes.c_int
        L.oracle_point_gen.argtypes = [ctypes.c_int, ctypes.c_int, _DP, ctypes.c_uint64,
                                       ctypes.c_int, i64, i64, i64, i64, i64, i64, _DP]
        L.oracle_point_gen.restype = ctypes.c_int
        for f in ("oracle_hypterm_flops", "oracle_rhs4_flops"):
            getattr(L, f).restype = i64
            getattr(L, f).argtypes = []
        for f in ("oracle_star_flops", "oracle_box_flops"):
            getattr(L, f).restype = i64
            getattr(L, f).argtypes = [ctypes.c_int]
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    assert a.dtype == np.float64 and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(_DP)


def sweep(kind: int, order: int, coeffs, layout: Layout, ins, outs, nsteps: int = 1,
          nthreads: int | None = None) -> None:
    """Run the definition in place on flat padded buffers (see cstgen.Layout)."""
    c = np.ascontiguousarray(coeffs, dtype=np.float64)
    nin, nout = N_IN[kind], N_OUT[kind]
    assert len(ins) == nin and len(outs) == nout
    pin = (_DP * nin)(*[_ptr(a) for a in ins])
    pout = (_DP * nout)(*[_ptr(a) for a in outs])
    L = layout
    rc = lib().oracle_sweep(kind, order, _ptr(c), L.nx, L.ny, L.nz, L.halo, L.lead_x,
                            L.pitch_x, L.pitch_y, pin, pout, nsteps,
                            nthreads or os.cpu_count() or 1)
    if rc != 0:
        raise ValueError(f"oracle_sweep rejected arguments (rc={rc})")


def point_gen(kind: int, order: int, coeffs, seed: int, array_id0: int, nx: int, ny: int,
              halo: int, x: int, y: int, z: int) -> np.ndarray:
    """One output point (all outputs) with inputs taken from the generator at global coords."""
    c = np.ascontiguousarray(coeffs, dtype=np.float64)
    out = np.zeros(5, dtype=np.float64)
    rc = lib().oracle_point_gen(kind, order, _ptr(c), seed, array_id0, nx, ny, halo, x, y, z,
                                _ptr(out))
    if rc != 0:
        raise ValueError("oracle_point_gen rejected arguments")
    return out[: N_OUT[kind]].copy()


def hypterm_flops() -> int:
    return int(lib().oracle_hypterm_flops())


def rhs4_flops() -> int:
    return int(lib().oracle_rhs4_flops())


def star_flops(r: int) -> int:
    return int(lib().oracle_star_flops(r))


def box_flops(r: int) -> int:
    return int(lib().oracle_box_flops(r))


# ---- coefficient sets of the configs (readings Q1, Q5) --------------------

# Central second-derivative weights of radius r (integer numerators, denominator D).
D2_INT = {
    1: ([1, -2, 1], 1),
    2: ([-1, 16, -30, 16, -1], 12),
    3: ([2, -27, 270, -490, 270, -27, 2], 180),
    4: ([-9, 128, -1008, 8064, -14350, 8064, -1008, 128, -9], 5040),
}


def star_laplacian_coeffs(r: int, integer: bool = False) -> np.ndarray:
    """[c0, wx[-r..-1], wx[1..r], wy.., wz..] for the FD Laplacian; c0 = 3 w[0]."""
    w, D = D2_INT[r]
    w = np.array(w, dtype=np.float64)
    if not integer:
        w = w / D
    side = np.concatenate([w[:r], w[r + 1:]])
    return np.concatenate([[3 * w[r]], side, side, side])


def box_binomial_coeffs() -> np.ndarray:
    b = np.array([0.25, 0.5, 0.25])
    return np.einsum("i,j,k->ijk", b, b, b).reshape(-1)


HYPTERM_A = (4.0 / 5.0, -1.0 / 5.0, 4.0 / 105.0, -1.0 / 280.0)
HYPTERM_A_INT = (672.0, -168.0, 32.0, -3.0)


def hypterm_coeffs(integer: bool = False, dxinv=(1.0, 1.0, 1.0)) -> np.ndarray:
    a = HYPTERM_A_INT if integer else HYPTERM_A
    return np.array(list(a) + list(dxinv), dtype=np.float64)


def rhs4_coeffs(scales=(1.0, 1.0, 1.0)) -> np.ndarray:
    return np.array(scales, dtype=np.float64)
