"""Pins for the oracle's one-sided (position-dependent) kernel near non-periodic boundaries
("an asymmetric (one-sided) stencil is used [21]";
ref [21] Ryan & Shu 2003, L1085; reading R4).

Reading R4: on a non-periodic axis [a, b] the 2k+1 B-spline nodes move to x_g = -k + g + lambda,
lambda(x) = max(0, H - (x-a)/h) + min(0, (b-x)/h - H), H = (3k+1)/2, so the support
x + h[-H + lambda, H + lambda] stays inside [a, b]; the coefficients re-solve the symmetric
kernel's moment conditions at the shifted nodes.  What pins it (none of it re-types the solve):
  * k = 1 closed form of c(lambda), solved by hand below;
  * lambda = 0 gives the classical symmetric coefficients;
  * the kernel evaluated by the C core has moments delta_m0 (m <= 2k) and its support is the
    shifted interval (Gauss quadrature per unit cell, exact for the pieces);
  * u = 1 -> u* = 1 with integrated area W^2 at every point up to the corners (no zero extension);
  * every polynomial of degree <= 2k per axis is reproduced at EVERY point, including the
    boundary and the corners (the property the one-sided kernel exists for); degree 2k+1 is
    not reproduced near the boundary (negative control) but is in the interior;
  * an exact-rational brute force (tests/exact_siac.py) whose coefficients come from a
    different formula: the shifted kernel is the symmetric-grid kernel with moments
    (-lambda)^m, c = A^{-1} (1, -lambda, lambda^2, ...).
"""
import math
from fractions import Fraction as Fr

import numpy as np
import pytest

from paper_conf_sc_0007k13_b200 import inputs

from exact_siac import exact_siac


def test_k1_closed_form():
    """k = 1, nodes (lam-1, lam, lam+1), hat functions (second moment 1/6):
    sum c = 1, sum c x = 0, sum c (x^2 + 1/6) = 0  =>  c = ((lam^2 + lam - 1/6)/2, 7/6 - lam^2,
    (lam^2 - lam - 1/6)/2)."""
    import oracle
    for lam in (Fr(0), Fr(1, 2), Fr(2), Fr(-3, 7), Fr(0.3125)):
        c = oracle.kernel_coefficients_shifted(1, lam)
        assert c == [(lam * lam + lam - Fr(1, 6)) / 2, Fr(7, 6) - lam * lam, (lam * lam - lam - Fr(1, 6)) / 2]


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_lambda_zero_is_symmetric(k):
    import oracle
    assert oracle.kernel_coefficients_shifted(k, 0.0) == oracle.kernel_coefficients(k)


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_shifted_kernel_moments_and_support(k):
    import oracle
    H = 0.5 * (3 * k + 1)
    g, wg = np.polynomial.legendre.leggauss(k + 6)
    for lam in (0.0, 0.37, 1.5, H, -2.25):
        c = oracle.kernel_coefficients_shifted(k, lam)
        lo = -H + lam
        cells = [(lo + i, lo + i + 1) for i in range(3 * k + 1)]
        t = np.concatenate([0.5 * (a + b) + 0.5 * g for a, b in cells])
        w = np.concatenate([0.5 * wg for _ in cells])
        K = oracle.kernel_values_shifted(k, c, lam, t)
        scale = max(1.0, max(abs(float(v)) for v in c))
        for m in range(2 * k + 1):
            mom = float(np.sum(w * K * t ** m))
            assert abs(mom - (1.0 if m == 0 else 0.0)) < 1e-12 * scale * (1 + abs(lam)) ** m, (lam, m, mom)
        outside = np.array([lo - 0.3, lo - 1e-9, lo + 3 * k + 1 + 1e-9, lo + 3 * k + 1.7])
        assert np.all(oracle.kernel_values_shifted(k, c, lam, outside) == 0.0)


def onesided_tol(k, h, P, periodic=0):
    """Rounding bound of a one-sided evaluation at each point: the shifted kernels' coefficients
    grow with lambda (sum |c| = 1.3 / 6.7 / 57 / 558 / 5848 for k = 1..4 at full shift), and
    u* = sum_{g,d} c_g c_d (integrals of O(1)) cancels down to O(1), so the error is of order
    eps * (sum |c_x|)(sum |c_y|) (reading R4); plus 1e-13 for the symmetric part."""
    import oracle
    S = np.ones((len(P), 2))
    for ax in (0, 1):
        if not periodic & (1 << ax):
            lam = oracle.onesided_shift(k, h, P[:, ax], 0.0, 1.0)
            S[:, ax] = [sum(abs(float(c)) for c in oracle.kernel_coefficients_shifted(k, float(l))) for l in lam]
    return 1e-13 + 1e-15 * S[:, 0] * S[:, 1]


def _boundary_points(k, h, n_inner=6):
    """Points on the boundary, at the corners, just inside, and a few interior ones."""
    H = 0.5 * (3 * k + 1) * h
    P = [[0, 0], [1, 1], [0, 1], [1, 0], [0, 0.5], [0.5, 1], [1e-3, 0.31], [0.999, 0.73],
         [0.5 * H, 0.5], [0.5, 1 - 0.3 * H], [H * 0.999, H * 1.001], [0.42, 0.0]]
    P += np.random.default_rng(k).uniform(H + 0.01, 1 - H - 0.01, (n_inner, 2)).tolist()
    return np.array(P, dtype=np.float64)


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_constant_field_every_point(oracle_mod, k):
    V, T = inputs.lattice_delaunay_mesh(900, seed=31)
    h = 0.05
    C = np.zeros((len(T), inputs.n_modes(k)))
    C[:, 0] = math.sqrt(2.0)
    P = _boundary_points(k, h)
    for per in (0, 1, 2):
        u, area = oracle_mod.oracle_eval(V, T, C, k, h, P, periodic=per, boundary=1, return_area=True)
        assert np.all(np.abs(u - 1) < onesided_tol(k, h, P, per))
        assert np.abs(area - ((3 * k + 1) * h) ** 2).max() < 1e-13


@pytest.mark.parametrize("k", [1, 2, 3])
def test_monomial_reproduction_up_to_the_boundary(oracle_mod, k):
    """x^a y^b with a, b <= 2k reproduced at boundary and corner points; a = 2k+1 is not
    reproduced at boundary points (the shifted kernel's odd moments do not vanish) but is at
    interior points (symmetric kernel there)."""
    V, T = inputs.lattice_delaunay_mesh(500, seed=32)
    h = 0.06
    P = _boundary_points(k, h, n_inner=3)
    H = 0.5 * (3 * k + 1) * h
    inner = np.all((P > H + 1e-9) & (P < 1 - H - 1e-9), axis=1)
    d = 2 * k + 1
    tol = onesided_tol(k, h, P)
    for a, b in [(0, 0), (2 * k, 0), (1, 2 * k), (2 * k, 2 * k), (d, 0)]:
        A = np.zeros((d + 1, d + 1))
        A[a, b] = 1.0
        u = oracle_mod.oracle_eval(V, T, A, k, h, P, periodic=0, field_mode=1, field_deg=d, boundary=1)
        exact = P[:, 0] ** a * P[:, 1] ** b
        if a <= 2 * k and b <= 2 * k:
            assert np.all(np.abs(u - exact) < tol), (a, b)
        else:
            assert np.abs(u - exact)[inner].max() < 1e-12
            assert np.abs(u - exact)[~inner].max() > 1e3 * tol[~inner].max()


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_dg_polynomial_reproduction_up_to_the_boundary(oracle_mod, k):
    V, T = inputs.lattice_delaunay_mesh(800, seed=33)
    f = lambda x, y: 0.2 + (x - 0.3 * y) ** k - 0.7 * x * y ** (k - 1)  # noqa: E731
    C = inputs.project(V, T, k, f)
    h = 0.04
    P = _boundary_points(k, h)
    u = oracle_mod.oracle_eval(V, T, C, k, h, P, periodic=0, boundary=1)
    assert np.all(np.abs(u - f(P[:, 0], P[:, 1])) < onesided_tol(k, h, P))
    uz = oracle_mod.oracle_eval(V, T, C, k, h, P, periodic=0, boundary=0)
    assert np.abs(uz - f(P[:, 0], P[:, 1])).max() > 1e-2          # zero extension does not


def _coeffs_by_moment_identity(k, lam):
    """c(lambda) = A^{-1} b, b_m = (-lambda)^m, A[m][g] = int psi(t - (g-k)) t^m dt: the
    shifted kernel written on the symmetric node grid (K_lam(t) = Kt(t - lam) with Kt's moments
    (-lam)^m).  Exact rationals; a different route from the oracle's shifted-node solve."""
    import oracle
    n = 2 * k + 1
    mu = [oracle.bspline_moments(k, l) for l in range(n)]
    A = [[sum(math.comb(m, l) * Fr(g - k) ** (m - l) * mu[l] for l in range(m + 1)) for g in range(n)]
         for m in range(n)]
    b = [(-Fr(lam)) ** m for m in range(n)]
    M = [A[i][:] + [b[i]] for i in range(n)]
    for col in range(n):                     # plain elimination, back substitution
        piv = next(r for r in range(col, n) if M[r][col] != 0)
        M[col], M[piv] = M[piv], M[col]
        for r in range(col + 1, n):
            f = M[r][col] / M[col][col]
            M[r] = [x - f * y for x, y in zip(M[r], M[col])]
    c = [Fr(0)] * n
    for i in reversed(range(n)):
        c[i] = (M[i][n] - sum(M[i][j] * c[j] for j in range(i + 1, n))) / M[i][i]
    return c


def test_moment_identity_matches_shifted_solve():
    import oracle
    for k in (1, 2, 3):
        for lam in (Fr(1, 3), Fr(5, 2), Fr(-7, 4)):
            assert _coeffs_by_moment_identity(k, lam) == oracle.kernel_coefficients_shifted(k, lam)


def _tiny_mesh():
    n = 3
    V = [[Fr(i, n), Fr(j, n)] for j in range(n + 1) for i in range(n + 1)]
    moves = {(1, 1): (Fr(1, 17), Fr(-1, 23)), (2, 1): (Fr(-1, 19), Fr(1, 29)),
             (1, 2): (Fr(1, 31), Fr(1, 13)), (2, 2): (Fr(-1, 11), Fr(-1, 37))}
    for (i, j), (dx, dy) in moves.items():
        V[j * (n + 1) + i][0] += dx
        V[j * (n + 1) + i][1] += dy
    _, T = inputs.structured_mesh(n)
    return V, T.tolist()


@pytest.mark.parametrize("k,h,pts", [
    (1, Fr(1, 5), [(Fr(1, 7), Fr(2, 9)), (Fr(19, 20), Fr(1, 2)), (Fr(0), Fr(1))]),
    (2, Fr(1, 8), [(Fr(3, 7), Fr(1, 16)), (Fr(1, 40), Fr(97, 100))]),
])
def test_exact_rational_brute_force_onesided(oracle_mod, k, h, pts):
    """Non-periodic tiny mesh, points near edges and corners: the oracle (shifted nodes, Cox-de
    Boor, slab/strip Gauss) against exact rational integration of the truncated-power kernel
    with coefficients from the moment identity at the effective point x + lambda h."""
    Vq, Tl = _tiny_mesh()
    rng = np.random.default_rng(70 + k)
    mons = [(a, b) for a in range(k + 1) for b in range(k + 1 - a)]
    fields = [{m: Fr(int(rng.integers(-9, 10)), int(rng.integers(1, 7))) for m in mons} for _ in Tl]
    Hh = Fr(3 * k + 1, 2) * h
    exact = []
    for x in pts:
        lam = [max(Fr(0), (Hh - x[ax]) / h) + min(Fr(0), (1 - x[ax] - Hh) / h) for ax in (0, 1)]
        xe = (x[0] + lam[0] * h, x[1] + lam[1] * h)
        exact.append(exact_siac(Vq, Tl, fields, k, h, _coeffs_by_moment_identity(k, lam[0]), xe, periodic=0,
                                coeffs_y=_coeffs_by_moment_identity(k, lam[1])))
    V = np.array([[float(a), float(b)] for a, b in Vq])
    T = np.array(Tl, dtype=np.int32)
    cf = np.array([[float(fl[m]) for m in mons] for fl in fields])

    def f(X, Y):
        return sum(cf[:, i][:, None] * X ** a * Y ** b for i, (a, b) in enumerate(mons))

    C = inputs.project(V, T, k, f)
    u = oracle_mod.oracle_eval(V, T, C, k, float(h), np.array([[float(a), float(b)] for a, b in pts]),
                               periodic=0, boundary=1)
    ex = np.array([float(e) for e in exact])
    P = np.array([[float(a), float(b)] for a, b in pts])
    assert np.all(np.abs(u - ex) < onesided_tol(k, float(h), P) * max(1.0, np.abs(ex).max()))


def test_interior_points_unchanged(oracle_mod):
    """lambda = 0 away from the boundary: the one-sided and zero-extension evaluations agree
    bitwise there (the same kernel, the same pieces)."""
    w = inputs.make_config(2, field_kind="random")
    P = w.points[::97]
    H = 0.5 * (3 * w.k + 1) * w.h
    inner = np.all((P > H) & (P < 1 - H), axis=1)
    u1 = oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, P[inner], periodic=0, boundary=1)
    u0 = oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, P[inner], periodic=0, boundary=0)
    assert inner.sum() > 10 and np.array_equal(u0, u1)
