"""Helpers for GPU parity tests: oracle on cstgen inputs vs libcst on the same inputs."""
from __future__ import annotations

import numpy as np

import cstgen
from oracle import stencil as ost

TOL = 1e-12   # north_star: 1e-12 relative max-norm (covers FMA contraction + reordering)


def coeffs(kind, r, variant="config", seed=0):
    if variant == "random":
        rng = np.random.default_rng(1000 + seed)
        n = {1: 6 * r + 1, 2: 27, 3: 7, 4: 3}[kind]
        c = rng.uniform(-1, 1, n)
        if kind == 3:
            c[4:] = rng.uniform(0.5, 2.0, 3)
        if kind == 4:
            c = rng.uniform(0.5, 2.0, 3)
        return c
    if kind == 1:
        return ost.star_laplacian_coeffs(r)
    if kind == 2:
        return ost.box_binomial_coeffs()
    if kind == 4:
        return ost.rhs4_coeffs()
    return ost.hypterm_coeffs()


def layout(n, halo):
    nx, ny, nz = n
    return cstgen.make_layout(nx, ny, nz, halo)


def inputs(kind, L, seed, poison_beyond=None):
    """cstgen inputs; cells farther than `poison_beyond` from the interior become NaN."""
    ins = [cstgen.fill(L, seed=seed, array_id=a) for a in range(ost.N_IN[kind])]
    if poison_beyond is not None and poison_beyond < L.halo:
        for b in ins:
            v = L.view(b)
            h, p = L.halo, poison_beyond
            m = np.ones(v.shape, bool)
            m[h - p:h + L.nz + p, h - p:h + L.ny + p, h - p:h + L.nx + p] = False
            v[m] = np.nan
    return ins


def oracle_outputs(kind, r, c, L, ins, nsteps=1):
    ins = [b.copy() for b in ins]
    outs = [np.full(L.numel, np.nan) for _ in range(ost.N_OUT[kind])]
    if nsteps > 1:
        # ping-pong: the output buffer's halo holds Dirichlet data too (= input halo here)
        outs = [b.copy() for b in ins]
        for o in outs:
            h = L.halo
            L.view(o)[h:h + L.nz, h:h + L.ny, h:h + L.nx] = np.nan
    ost.sweep(kind, r, c, L, ins, outs, nsteps=nsteps)
    return ins, outs


def interior(L, buf):
    h = L.halo
    return L.view(buf)[h:h + L.nz, h:h + L.ny, h:h + L.nx]


def assert_parity(L, got, want, what=""):
    gi, wi = interior(L, got), interior(L, want)
    assert np.all(np.isfinite(gi)), f"{what}: non-finite interior values (out-of-range read?)"
    scale = np.max(np.abs(wi))
    err = np.max(np.abs(gi - wi))
    if scale == 0:
        assert err == 0, what
    else:
        assert err <= TOL * scale, f"{what}: max err {err:.3e} vs {TOL * scale:.3e}"
    return err / scale if scale else 0.0


def assert_halo_untouched(L, got, before):
    g = got.copy()
    b = before.copy()
    gi = interior(L, g)
    bi = interior(L, b)
    gi[...] = 0
    bi[...] = 0
    assert np.array_equal(g.view(np.uint64), b.view(np.uint64)), "halo / pad bytes changed"
