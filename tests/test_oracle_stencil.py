"""Pins of the stencil oracle (oracle/oracle.cpp) against what the definitions and the
paper fix — never against a re-typing of the oracle's own formula.  CPU only.

* polynomial exactness of FD weights of radius r (north_star: "finite-difference weights
  of order k reproduce polynomials of degree <= k exactly"), incl. tightness;
* constant fields give exactly zero for derivative stencils (north_star);
* hand-computed values on 4^3 grids (north_star);
* impulse responses = (reflected) coefficient tables;
* a library routine: scipy.ndimage.correlate with the (2r+1)^3 kernel;
* hypterm-like: -840 x analytic divergence of polynomial fields (sympy), constant
  fields -> 0, and the Table III FLOP count (358).
"""
import numpy as np
import pytest
import scipy.ndimage
import sympy as sp

import cstgen
from oracle import stencil as ost


def grid_from(fn, n, halo, nz=None, dtype=np.float64):
    nz = n if nz is None else nz
    L = cstgen.make_layout(n, n, nz, halo)
    buf = np.full(L.numel, np.nan)
    v = L.view(buf)
    r = np.arange(-halo, n + halo)
    rz = np.arange(-halo, nz + halo)
    Z, Y, X = np.meshgrid(rz, r, r, indexing="ij")
    v[...] = fn(X.astype(dtype), Y.astype(dtype), Z.astype(dtype))
    return L, buf


def run(kind, r, c, L, ins, nsteps=1):
    outs = [np.full(L.numel, np.nan) for _ in range(ost.N_OUT[kind])]
    ost.sweep(kind, r, c, L, ins, outs, nsteps=nsteps)
    return outs


def interior(L, buf):
    h = L.halo
    return L.view(buf)[h:h + L.nz, h:h + L.ny, h:h + L.nx]


# ------------------------------------------------------------------ star, integer form
@pytest.mark.parametrize("r,D", [(2, 12), (4, 5040)])
def test_star_quadratic_and_constant(r, D):
    c = ost.star_laplacian_coeffs(r, integer=True)
    L, u = grid_from(lambda x, y, z: x * x, 4, r)
    out = interior(L, run(ost.STAR, r, c, L, [u])[0])
    assert np.all(out == 2 * D)                    # D * d2/dx2 x^2
    L, u = grid_from(lambda x, y, z: 0 * x + 3.0, 4, r)
    assert np.all(interior(L, run(ost.STAR, r, c, L, [u])[0]) == 0.0)


def test_star_r2_hand_values_4cubed():
    # u = x^4: 12 * 12 x^2 = 144 x^2 -> (0, 144, 576, 1296) along x (hand-computed)
    c = ost.star_laplacian_coeffs(2, integer=True)
    L, u = grid_from(lambda x, y, z: x ** 4, 4, 2)
    out = interior(L, run(ost.STAR, 2, c, L, [u])[0])
    assert np.all(out == np.array([0.0, 144.0, 576.0, 1296.0])[None, None, :])
    # u = x^2 y^2: 12 * (2 y^2 + 2 x^2) = 24 (x^2 + y^2)
    L, u = grid_from(lambda x, y, z: x * x * y * y, 4, 2)
    out = interior(L, run(ost.STAR, 2, c, L, [u])[0])
    xs = np.arange(4.0)
    assert np.array_equal(out, np.broadcast_to(24 * (xs[None, :] ** 2 + xs[:, None] ** 2), (4, 4, 4)))


def test_star_r4_hand_values():
    c = ost.star_laplacian_coeffs(4, integer=True)
    L, u = grid_from(lambda x, y, z: x ** 4, 4, 4)
    out = interior(L, run(ost.STAR, 4, c, L, [u])[0])
    assert np.all(out == np.array([0.0, 60480.0, 241920.0, 544320.0])[None, None, :])


@pytest.mark.parametrize("r,D,axis", [(2, 12, 0), (2, 12, 2), (4, 5040, 1), (4, 5040, 2)])
def test_star_degree_bound_is_tight(r, D, axis):
    """Radius-r D2 weights are exact up to degree 2r+1 and fail at 2r+2 (Q2)."""
    c = ost.star_laplacian_coeffs(r, integer=True)
    sel = lambda x, y, z: (x, y, z)[axis]
    p = 2 * r + 1
    L, u = grid_from(lambda x, y, z: sel(x, y, z) ** p, 4, r)
    out = interior(L, run(ost.STAR, r, c, L, [u])[0])
    t = np.arange(4.0)
    want = D * p * (p - 1) * t ** (p - 2)
    shape = [1, 1, 1]
    shape[2 - axis] = 4
    assert np.array_equal(out, np.broadcast_to(want.reshape(shape), (4, 4, 4)))
    L, u = grid_from(lambda x, y, z: sel(x, y, z) ** (p + 1), 4, r)
    out = interior(L, run(ost.STAR, r, c, L, [u])[0])
    want = D * (p + 1) * p * t ** (p - 1)
    assert not np.array_equal(out, np.broadcast_to(want.reshape(shape), (4, 4, 4)))


@pytest.mark.parametrize("r,n", [(2, 8), (4, 12)])
def test_star_impulse_response(r, n):
    c = ost.star_laplacian_coeffs(r, integer=True)
    ctr = n // 2
    L, u = grid_from(lambda x, y, z: ((x == ctr) & (y == ctr) & (z == ctr)).astype(float), n, r)
    out = interior(L, run(ost.STAR, r, c, L, [u])[0])
    w, _ = ost.D2_INT[r]
    assert np.count_nonzero(out) == 6 * r + 1
    assert out[ctr, ctr, ctr] == 3 * w[r]
    for k in range(-r, r + 1):
        if k == 0:
            continue
        # out(p) picks w[k] u(p + k e) -> impulse seen at p = ctr - k
        assert out[ctr, ctr, ctr - k] == w[k + r]
        assert out[ctr, ctr - k, ctr] == w[k + r]
        assert out[ctr - k, ctr, ctr] == w[k + r]


def _star_kernel(r, c):
    K = np.zeros((2 * r + 1,) * 3)
    K[r, r, r] = c[0]
    idx = 1
    for axis in range(3):                       # x, y, z ; K is [dz][dy][dx]
        for k in list(range(-r, 0)) + list(range(1, r + 1)):
            pos = [r, r, r]
            pos[2 - axis] = r + k
            K[tuple(pos)] = c[idx]
            idx += 1
    return K


@pytest.mark.parametrize("kind,r", [(ost.STAR, 1), (ost.STAR, 2), (ost.STAR, 3), (ost.STAR, 4), (ost.BOX, 1)])
def test_random_coeffs_match_scipy_correlate(kind, r):
    """Library routine pin: a star/box stencil is the correlation of the padded input with
    its (2r+1)^3 coefficient kernel, restricted to the interior."""
    rng = np.random.default_rng(10 + r + kind)
    n, nz = 9, 7
    L = cstgen.make_layout(n, n, nz, r)
    u = cstgen.fill(L, seed=5, array_id=0)
    if kind == ost.STAR:
        c = rng.uniform(-1, 1, 6 * r + 1)
        K = _star_kernel(r, c)
    else:
        c = rng.uniform(-1, 1, 27)
        K = c.reshape(3, 3, 3)
    out = interior(L, run(kind, r, c, L, [u])[0])
    ref = scipy.ndimage.correlate(L.view(u), K, mode="constant", cval=0.0)
    ref = ref[r:r + nz, r:r + n, r:r + n]
    assert np.max(np.abs(out - ref)) <= 1e-13 * np.max(np.abs(ref))


# ------------------------------------------------------------------ box binomial
def test_box_binomial_pins():
    c = ost.box_binomial_coeffs()
    L, u = grid_from(lambda x, y, z: 0 * x + 0.75, 4, 1)
    assert np.all(interior(L, run(ost.BOX, 1, c, L, [u])[0]) == 0.75)
    L, u = grid_from(lambda x, y, z: x + 2 * y + 3 * z, 4, 1)
    out = interior(L, run(ost.BOX, 1, c, L, [u])[0])
    t = np.arange(4.0)
    assert np.array_equal(out, t[None, None, :] + 2 * t[None, :, None] + 3 * t[:, None, None])
    L, u = grid_from(lambda x, y, z: x * x, 4, 1)
    out = interior(L, run(ost.BOX, 1, c, L, [u])[0])
    assert np.all(out == np.array([0.5, 1.5, 4.5, 9.5])[None, None, :])
    ctr = 3
    L, u = grid_from(lambda x, y, z: ((x == ctr) & (y == ctr) & (z == ctr)).astype(float), 6, 1)
    out = interior(L, run(ost.BOX, 1, c, L, [u])[0])
    blk = out[ctr - 1:ctr + 2, ctr - 1:ctr + 2, ctr - 1:ctr + 2]
    assert np.count_nonzero(out) == 27
    assert np.array_equal(blk, c.reshape(3, 3, 3)[::-1, ::-1, ::-1])
    assert sorted(set(blk.ravel().tolist())) == [1 / 64, 1 / 32, 1 / 16, 1 / 8]


# ------------------------------------------------------------------ hypterm-like
def test_hypterm_flop_count_matches_table3():
    assert ost.hypterm_flops() == 358          # Table III
    assert ost.star_flops(4) == 49 and ost.star_flops(2) == 25
    assert ost.box_flops(1) == 53


def test_hypterm_constant_fields_zero_with_real_weights():
    c = ost.hypterm_coeffs(integer=False, dxinv=(0.37, 1.9, 2.5))
    L = cstgen.make_layout(5, 5, 5, 4)
    ins = []
    for a in range(8):
        b = np.full(L.numel, np.nan)
        L.view(b)[...] = 0.1 + 0.3 * a
        ins.append(b)
    outs = run(ost.HYPTERM, 4, c, L, ins)
    for o in outs:
        assert np.all(interior(L, o) == 0.0)


def _hypterm_poly_case(seed, dxinv):
    rng = np.random.default_rng(seed)
    X, Y, Z = sp.symbols("x y z")
    mons = [1, X, Y, Z, X * X, Y * Y, Z * Z, X * Y, Y * Z, X * Z]
    fields = [sum(int(rng.integers(-3, 4)) * m for m in mons) for _ in range(8)]
    c1, c2, c3, c4, q1, q2, q3, q4 = fields
    dx, dy, dz = [sp.Integer(int(v)) for v in dxinv]
    div = lambda fx, fy, fz: dx * sp.diff(fx, X) + dy * sp.diff(fy, Y) + dz * sp.diff(fz, Z)
    want = [
        -840 * div(c1, c2, c3),
        -840 * div(c1 * q1 + q4, c1 * q2, c1 * q3),
        -840 * div(c2 * q1, c2 * q2 + q4, c2 * q3),
        -840 * div(c3 * q1, c3 * q2, c3 * q3 + q4),
        -840 * div(c4 * q1 + q4 * q1, c4 * q2 + q4 * q2, c4 * q3 + q4 * q3),
    ]
    return fields, want, (X, Y, Z)


@pytest.mark.parametrize("seed,dxinv", [(1, (1, 1, 1)), (2, (1, 2, 4)), (3, (4, 1, 2))])
def test_hypterm_polynomial_divergence(seed, dxinv):
    """Integer weights 840*a = (672,-168,32,-3), integer dxinv, degree<=2 fields (products
    degree<=4 <= 8): every output equals -840 x the analytic divergence, bit-exactly."""
    fields, want, (X, Y, Z) = _hypterm_poly_case(seed, dxinv)
    n, r = 4, 4
    c = ost.hypterm_coeffs(integer=True, dxinv=dxinv)
    ins = []
    for f in fields:
        fn = sp.lambdify((X, Y, Z), f, "numpy")
        L, b = grid_from(lambda x, y, z: fn(x, y, z) + 0 * x, n, r)
        ins.append(b)
    outs = run(ost.HYPTERM, 4, c, L, ins)
    t = np.arange(n, dtype=np.float64)
    Zg, Yg, Xg = np.meshgrid(t, t, t, indexing="ij")
    for o, w in zip(outs, want):
        fn = sp.lambdify((X, Y, Z), w, "numpy")
        ref = fn(Xg, Yg, Zg) + 0 * Xg
        assert np.array_equal(interior(L, o), ref)


# ------------------------------------------------------------------ sweep semantics
@pytest.mark.parametrize("kind,r", [(ost.STAR, 2), (ost.BOX, 1), (ost.HYPTERM, 4)])
def test_output_halos_untouched_and_inputs_read_only_in_range(kind, r):
    n = 6
    L = cstgen.make_layout(n, n, n, r)
    ins = [cstgen.fill(L, seed=9, array_id=a) for a in range(ost.N_IN[kind])]
    c = {ost.STAR: ost.star_laplacian_coeffs(r), ost.BOX: ost.box_binomial_coeffs(),
         ost.HYPTERM: ost.hypterm_coeffs()}[kind]
    outs = run(kind, r, c, L, ins)
    for o in outs:
        v = L.view(o)
        h = L.halo
        assert np.all(np.isfinite(interior(L, o)))
        mask = np.ones(v.shape, bool)
        mask[h:h + n, h:h + n, h:h + n] = False
        assert np.all(np.isnan(v[mask]))        # halo never written (pads are NaN too)


def test_multistep_is_composition_and_halos_fixed():
    r, n = 2, 6
    c = ost.star_laplacian_coeffs(r)
    L = cstgen.make_layout(n, n, n, r)
    a = cstgen.fill(L, seed=1, array_id=0)
    b = cstgen.fill(L, seed=1, array_id=1)
    a0, b0 = a.copy(), b.copy()
    ost.sweep(ost.STAR, r, c, L, [a], [b], nsteps=3)   # result in b (odd)
    # compose three single steps by hand
    x, y = a0.copy(), b0.copy()
    ost.sweep(ost.STAR, r, c, L, [x], [y], nsteps=1)
    ost.sweep(ost.STAR, r, c, L, [y], [x], nsteps=1)
    ost.sweep(ost.STAR, r, c, L, [x], [y], nsteps=1)
    assert np.array_equal(b, y, equal_nan=True) and np.array_equal(a, x, equal_nan=True)
    h = L.halo
    for cur, orig in ((a, a0), (b, b0)):
        v, v0 = L.view(cur), L.view(orig)
        mask = np.ones(v.shape, bool)
        mask[h:h + n, h:h + n, h:h + n] = False
        assert np.array_equal(v[mask], v0[mask])


@pytest.mark.parametrize("kind,r", [(ost.STAR, 4), (ost.BOX, 1), (ost.HYPTERM, 4)])
def test_point_gen_equals_sweep_on_generated_grid(kind, r):
    n = 6
    L = cstgen.make_layout(n, n, n, r)
    ins = [cstgen.fill(L, seed=21, array_id=a) for a in range(ost.N_IN[kind])]
    c = {ost.STAR: ost.star_laplacian_coeffs(r), ost.BOX: ost.box_binomial_coeffs(),
         ost.HYPTERM: ost.hypterm_coeffs()}[kind]
    outs = run(kind, r, c, L, ins)
    for (x, y, z) in [(0, 0, 0), (5, 5, 5), (2, 4, 1)]:
        p = ost.point_gen(kind, r, c, 21, 0, n, n, r, x, y, z)
        for o in range(ost.N_OUT[kind]):
            assert p[o] == outs[o][L.offset(x, y, z)]


def test_invalid_arguments_rejected():
    L = cstgen.make_layout(4, 4, 4, 1)
    u = np.zeros(L.numel)
    with pytest.raises(ValueError):
        ost.sweep(ost.STAR, 2, ost.star_laplacian_coeffs(2), L, [u], [u.copy()])  # halo < order
    with pytest.raises(ValueError):
        ost.sweep(ost.BOX, 2, np.zeros(125), L, [u], [u.copy()])                   # box r != 1


# ------------------------------------------------------------------ rhs4center-like (NEXT-1)
def test_rhs4_flop_count_matches_table3():
    assert ost.rhs4_flops() == 666          # Table III "rhs4center": 666 FLOPs


def _rhs4_run(fields, n=5, scales=(1.0, 1.0, 1.0)):
    X, Y, Z = sp.symbols("x y z")
    ins = []
    for f in fields:
        fn = sp.lambdify((X, Y, Z), f, "numpy")
        L, b = grid_from(lambda x, y, z: fn(x, y, z) + 0 * x, n, 2)
        ins.append(b)
    return L, run(ost.RHS4, 2, ost.rhs4_coeffs(scales), L, ins)


def _elastic(u, mu, la, X, Y, Z, scales=(1, 1, 1)):
    """Continuum d_j(mu (d_j u_i + d_i u_j)) + d_i(la div u) with x_d scaled by s_d."""
    xs = (X, Y, Z)
    D = lambda f, d: scales[d] * sp.diff(f, xs[d])
    div = sum(D(u[j], j) for j in range(3))
    return [sum(D(mu * (D(u[i], j) + D(u[j], i)), j) for j in range(3)) + D(la * div, i)
            for i in range(3)]


def test_rhs4_constant_fields_zero():
    L, outs = _rhs4_run([sp.Integer(3), sp.Integer(-2), sp.Integer(5), sp.Integer(2),
                         sp.Integer(7)])
    for o in outs:
        assert np.all(interior(L, o) == 0.0)


@pytest.mark.parametrize("seed,scales", [(1, (1, 1, 1)), (2, (1, 2, 0.5)), (3, (0.5, 1, 2))])
def test_rhs4_constant_coefficients_polynomial_exact(seed, scales):
    """Constant mu, lambda and displacements of total degree <= 4: the 4th-order operators
    reproduce mu lap u + (mu + la) grad div u up to rounding (closed form via sympy)."""
    rng = np.random.default_rng(seed)
    X, Y, Z = sp.symbols("x y z")
    mons = [X ** a * Y ** b * Z ** c for a in range(5) for b in range(5) for c in range(5)
            if a + b + c <= 4]
    u = [sum(int(rng.integers(-3, 4)) * m for m in rng.choice(mons, 8, replace=False))
         for _ in range(3)]
    mu, la = sp.Integer(3), sp.Integer(2)
    L, outs = _rhs4_run(u + [mu, la], scales=scales)
    want = _elastic(u, mu, la, X, Y, Z, scales)
    t = np.arange(5, dtype=np.float64)
    Zg, Yg, Xg = np.meshgrid(t, t, t, indexing="ij")
    for o, w in zip(outs, want):
        ref = sp.lambdify((X, Y, Z), w, "numpy")(Xg, Yg, Zg) + 0 * Xg
        got = interior(L, o)
        assert np.max(np.abs(got - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


def test_rhs4_degree_bound_is_tight():
    """The mixed terms use 4th-order first derivatives: degree 5 in the inner direction
    is no longer reproduced."""
    X, Y, Z = sp.symbols("x y z")
    u = [sp.Integer(0), X ** 5, sp.Integer(0)]            # u2 = x^5: d_y(mu d_x u2) ... and
    mu, la = sp.Integer(1), sp.Integer(1)                  # d_x(la d_y u2) = 0; d_x(mu d_x u2)
    L, outs = _rhs4_run(u + [mu, la])                      # is a 2nd derivative (exact to 5)
    t = np.arange(5, dtype=np.float64)
    Zg, Yg, Xg = np.meshgrid(t, t, t, indexing="ij")
    want = _elastic(u, mu, la, X, Y, Z)
    ref1 = sp.lambdify((X, Y, Z), want[1], "numpy")(Xg, Yg, Zg) + 0 * Xg
    assert np.max(np.abs(interior(L, outs[1]) - ref1)) <= 1e-9 * np.max(np.abs(ref1))
    u = [X * Y ** 5, sp.Integer(0), sp.Integer(0)]         # d_x(la d_x u1) ok, d_y(mu d_x u1)
    L, outs = _rhs4_run(u + [mu, la])                      # needs D_y of y^5 -> inexact
    want = _elastic(u, mu, la, X, Y, Z)
    ref1 = sp.lambdify((X, Y, Z), want[1], "numpy")(Xg, Yg, Zg) + 0 * Xg
    assert np.max(np.abs(interior(L, outs[1]) - ref1)) > 1e-6 * np.max(np.abs(ref1))


def test_rhs4_variable_coefficient_second_derivative():
    """Linear mu and quadratic u: d(mu du) is reproduced (the SW4 4th-order variable-
    coefficient operator is exact there); lambda = 0 so only the V and mu-mixed terms act."""
    X, Y, Z = sp.symbols("x y z")
    mu = 5 + X + 2 * Y - Z
    u = [X * X + Y * Z, Y * Y - X * Z, Z * Z + X * Y]
    L, outs = _rhs4_run(u + [mu, sp.Integer(0)], n=6)
    t = np.arange(6, dtype=np.float64)
    Zg, Yg, Xg = np.meshgrid(t, t, t, indexing="ij")
    for o, w in zip(outs, _elastic(u, mu, sp.Integer(0), X, Y, Z)):
        ref = sp.lambdify((X, Y, Z), w, "numpy")(Xg, Yg, Zg) + 0 * Xg
        assert np.max(np.abs(interior(L, o) - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))
