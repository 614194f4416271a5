"""cstgen.gen — numpy twin of cstgen/cst_gen.h.

Seeded, counter-based U[-1, 1) input generator shared by the oracle side and the
tests/bench.  It holds none of the stencil arithmetic.  Layout helpers here only
describe where grid element (x, y, z) lives in a padded, pitched buffer — the
C-ABI convention of include/cst.h:

    element (x, y, z), x, y, z in [-halo, n + halo):
        base[((z + halo) * pitch_y + (y + halo)) * pitch_x + lead_x + x]
"""
from __future__ import annotations

import dataclasses

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x):
    """Standard splitmix64 finaliser on a uint64 array (mod 2^64)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def key(seed: int, array_id: int) -> np.uint64:
    with np.errstate(over="ignore"):
        k = np.uint64(seed) ^ (np.uint64(array_id) * GOLDEN)
    return splitmix64(np.array([k], dtype=np.uint64))[0]


def value(k, g):
    """U[-1,1) value of stream key k at counter(s) g (exact in FP64)."""
    h = splitmix64(np.uint64(k) ^ np.asarray(g, dtype=np.uint64))
    return 2.0 * ((h >> np.uint64(11)).astype(np.float64) * 2.0 ** -53) - 1.0


def index(nx, ny, halo, x, y, z):
    """Global padded counter g for coordinates in [-halo, n + halo)."""
    x = np.asarray(x, dtype=np.int64)
    y = np.asarray(y, dtype=np.int64)
    z = np.asarray(z, dtype=np.int64)
    g = ((z + halo) * (ny + 2 * halo) + (y + halo)) * (nx + 2 * halo) + (x + halo)
    return g.astype(np.uint64)


def at(seed, array_id, nx, ny, halo, x, y, z):
    return value(key(seed, array_id), index(nx, ny, halo, x, y, z))


@dataclasses.dataclass(frozen=True)
class Layout:
    """Padded pitched grid (element counts).  nz is the number of LOCAL interior planes."""

    nx: int
    ny: int
    nz: int
    halo: int
    lead_x: int
    pitch_x: int
    pitch_y: int

    @property
    def planes(self) -> int:
        return self.nz + 2 * self.halo

    @property
    def numel(self) -> int:
        return self.planes * self.pitch_y * self.pitch_x

    def offset(self, x, y, z):
        return ((z + self.halo) * self.pitch_y + (y + self.halo)) * self.pitch_x + self.lead_x + x

    def view(self, buf: np.ndarray) -> np.ndarray:
        """[z][y][x] view of the logical padded region [-h, n+h)^3 of a flat buffer."""
        a = buf.reshape(self.planes, self.pitch_y, self.pitch_x)
        h = self.halo
        return a[:, : self.ny + 2 * h, self.lead_x - h : self.lead_x + self.nx + h]


def make_layout(nx, ny, nz, halo, lead_x=None, align=16) -> Layout:
    """Default layout: interior x=0 on a 128-B boundary (lead_x = 16 doubles when halo <= 16),
    row pitch rounded up to `align` doubles so every row starts 128-B aligned."""
    if lead_x is None:
        lead_x = max(16, -(-halo // 16) * 16)
    pitch_x = -(-(lead_x + nx + halo) // align) * align
    pitch_y = ny + 2 * halo
    return Layout(nx, ny, nz, halo, lead_x, pitch_x, pitch_y)


def fill(layout: Layout, seed: int, array_id: int, z0: int = 0, ny_global=None,
         nx_global=None, fill_pad=np.nan) -> np.ndarray:
    """Flat padded buffer whose logical region [-h, n+h)^3 holds generator values.

    `z0` is the global z of local interior plane 0 (z-slab decomposition); the counter
    uses the global extents.  Pad columns outside the logical region get `fill_pad`.
    """
    L = layout
    nxg = L.nx if nx_global is None else nx_global
    nyg = L.ny if ny_global is None else ny_global
    buf = np.full(L.numel, fill_pad, dtype=np.float64)
    v = L.view(buf)
    h = L.halo
    k = key(seed, array_id)
    xs = np.arange(-h, L.nx + h, dtype=np.int64)
    ys = np.arange(-h, L.ny + h, dtype=np.int64)
    for iz, z in enumerate(range(-h + z0, L.nz + h + z0)):
        g = index(nxg, nyg, h, xs[None, :], ys[:, None], z)
        v[iz] = value(k, g)
    return buf
