"""Pins of the counter-based input generator — CPU only."""
import json
import os

import numpy as np
import pytest

import cstgen
from oracle import stencil as ost

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "generator.json")


def test_splitmix64_reference_sequence():
    # SplitMix64 (Steele/Lea/Flood 2014) seeded with 0: the published first outputs.
    # Our splitmix64(x) = mix(x + golden) = output of a SplitMix64 whose state is x.
    g = 0x9E3779B97F4A7C15
    xs = np.array([0, g, (2 * g) % 2**64], dtype=np.uint64)
    assert [int(v) for v in cstgen.splitmix64(xs)] == [
        0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]


def test_generator_golden_values():
    with open(GOLDEN) as f:
        gold = json.load(f)
    for e in gold["values"]:
        v = cstgen.value(cstgen.key(e["seed"], e["array_id"]), np.array([e["g"]], dtype=np.uint64))[0]
        assert float(v).hex() == e["hex"], e


def test_generator_range_and_exactness():
    v = cstgen.value(cstgen.key(7, 3), np.arange(100000, dtype=np.uint64))
    assert v.min() >= -1.0 and v.max() < 1.0
    # v = 2*(m * 2^-53) - 1 with m < 2^53 integer: (v + 1) * 2^52 is an integer.
    m = (v + 1.0) * 2.0**52
    assert np.all(m == np.floor(m))
    assert abs(v.mean()) < 0.01


def test_c_twin_matches_numpy(oracle_lib):
    # The C twin (cst_gen.h, compiled into liboracle) is observed through a star stencil
    # whose only non-zero coefficient is c0 = 1, i.e. out(p) = u(p).
    c = np.zeros(13)
    c[0] = 1.0
    nx, ny, h = 5, 7, 2
    for (x, y, z) in [(0, 0, 0), (4, 6, 3), (2, 3, 100), (1, 5, 7)]:
        got = ost.point_gen(ost.STAR, 2, c, 11, 0, nx, ny, h, x, y, z)[0]
        want = cstgen.at(11, 0, nx, ny, h, x, y, z)
        assert got == want


def test_fill_layout_roundtrip():
    L = cstgen.make_layout(6, 5, 4, 2)
    buf = cstgen.fill(L, seed=3, array_id=1)
    v = L.view(buf)
    h = L.halo
    for (x, y, z) in [(-2, -2, -2), (0, 0, 0), (5, 4, 3), (7, 6, 5), (3, -1, 2)]:
        assert v[z + h, y + h, x + h] == cstgen.at(3, 1, 6, 5, 2, x, y, z)
        assert buf[L.offset(x, y, z)] == v[z + h, y + h, x + h]
    # slab fill: local plane 0 of a slab starting at global z0 equals global plane z0
    Ls = cstgen.make_layout(6, 5, 2, 2)
    slab = Ls.view(cstgen.fill(Ls, seed=3, array_id=1, z0=2))
    assert np.array_equal(slab, v[2:2 + 2 + 2 * h])
