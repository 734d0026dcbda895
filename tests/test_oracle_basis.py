"""Pins for the oracle's modal basis (SURVEY §8(b) basis convention, Q8; PAPER.md L716-718:
3/6/10 coefficients for P1/P2/P3, i.e. the full P_k basis)."""
import numpy as np
import pytest

from paper_conf_sc_0007k13_b200 import inputs


def _collapsed_rule(n):
    g, w = np.polynomial.legendre.leggauss(n)
    A, B = np.meshgrid(g, g, indexing="ij")
    WA, WB = np.meshgrid(w, w, indexing="ij")
    xi = (1 + A) * (1 - B) / 2 - 1
    return xi.ravel(), B.ravel(), (WA * WB * (1 - B) / 2).ravel()


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_dubiner_orthonormal(oracle_mod, k):
    """int_ref phi_i phi_j = delta_ij on {xi, eta >= -1, xi + eta <= 0}."""
    xi, eta, w = _collapsed_rule(k + 3)
    Phi = oracle_mod.dubiner_values(k, xi, eta)
    G = Phi.T @ (w[:, None] * Phi)
    assert np.abs(G - np.eye(len(G))).max() < 1e-13


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_dubiner_matches_scipy_jacobi(oracle_mod, k):
    """The oracle's recurrences vs an independent evaluation through scipy.special."""
    rng = np.random.default_rng(5)
    r, s = rng.uniform(0, 1, (2, 200))
    m = r + s > 1
    r[m], s[m] = 1 - r[m], 1 - s[m]
    xi, eta = 2 * r - 1, 2 * s - 1
    a = oracle_mod.dubiner_values(k, xi, eta)
    b = inputs.dubiner_eval(k, xi, eta)
    assert np.abs(a - b).max() < 1e-12


def test_dubiner_low_modes_closed_form(oracle_mod):
    """phi_00 = 1/sqrt 2, phi_10 = sqrt(3/2)*... written out: phi_10 = sqrt(3)(1 + 2 xi + eta)/sqrt(2)
    ... from the definition with p=1,q=0: sqrt(3*2/2) * (xi + (1+eta)/2)."""
    xi = np.array([-0.5, 0.1, -0.9])
    eta = np.array([-0.2, -0.6, 0.8])
    P = oracle_mod.dubiner_values(1, xi, eta)
    assert np.allclose(P[:, 0], 1 / np.sqrt(2), atol=1e-15)
    assert np.allclose(P[:, 1], np.sqrt(3.0) * (xi + (1 + eta) / 2), atol=1e-14)
    # p=0, q=1: sqrt(1*2/2) * P_1^(1,0)(eta) = (1 + 3 eta)/2
    assert np.allclose(P[:, 2], (1 + 3 * eta) / 2, atol=1e-14)


@pytest.mark.parametrize("k", [1, 2, 3])
def test_dubiner_at_top_vertex_finite(oracle_mod, k):
    """The collapsed recurrence has no division by (1 - eta): finite at eta = 1."""
    v = oracle_mod.dubiner_values(k, np.array([-1.0]), np.array([1.0]))
    assert np.all(np.isfinite(v))


# ------------------------------------------------------------------ SIAC_BASIS_MONOMIAL_REF
# (params.basis, "Sum c_ab r^a s^b on the unit reference triangle, offered for
# tests"; the oracle's field_mode 2)

def _mons(k):
    return [(n - b, b) for n in range(k + 1) for b in range(n + 1)]


def monomial_ref_coeffs(V, T, k, f):
    """Per-triangle coefficients of r^a s^b interpolating f at the lattice points (i/k, j/k)
    of the unit reference triangle (unisolvent for P_k): exact for f in P_k.  Input
    generation only (a Vandermonde solve), no SIAC arithmetic."""
    mons = _mons(k)
    rs = np.array([(i / k, j / k) for j in range(k + 1) for i in range(k + 1 - j)])
    A = np.stack([rs[:, 0] ** a * rs[:, 1] ** b for a, b in mons], axis=1)
    v0, v1, v2 = V[T[:, 0]], V[T[:, 1]], V[T[:, 2]]
    X = v0[:, None, :] + rs[None, :, 0, None] * (v1 - v0)[:, None, :] + rs[None, :, 1, None] * (v2 - v0)[:, None, :]
    F = f(X[..., 0], X[..., 1])
    return np.linalg.solve(A[None], F[..., None])[..., 0]


def monomial_to_dubiner(M, k, n_quad=None):
    """L2 projection onto the orthonormal Dubiner modes of sum_i M[t, i] r^a s^b (the input
    generator's collapsed rule and scipy Dubiner values; exact for degree k)."""
    xi, eta, W = inputs._ref_rule(n_quad or k + 2)
    Phi = inputs.dubiner_eval(k, xi, eta)
    r, s = (xi + 1) / 2, (eta + 1) / 2
    B = np.stack([r ** a * s ** b for a, b in _mons(k)], axis=1)       # (nq, nb)
    return ((M @ B.T) * W[None, :]) @ Phi


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_monomial_basis_reproduces_global_polynomial(oracle_mod, k):
    """u_h = a global polynomial of degree k written in per-triangle reference monomials ->
    u* = u at interior points (degree <= 2k reproduction, L202-205)."""
    V, T = inputs.lattice_delaunay_mesh(700, seed=8)
    f = lambda x, y: 0.3 - (x + 0.2 * y) ** k + 0.5 * x ** (k - 1) * y  # noqa: E731
    M = monomial_ref_coeffs(V, T, k, f)
    h = 0.03
    W = (3 * k + 1) * h
    P = np.random.default_rng(3).uniform(W / 2 + 0.01, 1 - W / 2 - 0.01, (10, 2))
    u = oracle_mod.oracle_eval(V, T, M, k, h, P, periodic=0, field_mode=2)
    assert np.abs(u - f(P[:, 0], P[:, 1])).max() < 1e-12


@pytest.mark.parametrize("k", [1, 3])
def test_monomial_basis_equals_dubiner_random_field(oracle_mod, k):
    """A random per-triangle field in reference monomials == the same field projected onto
    the Dubiner basis (two independent field evaluations inside the oracle)."""
    w = inputs.make_config(2)
    V, T = w.V, w.T
    M = np.random.default_rng(4).uniform(-1, 1, (len(T), inputs.n_modes(k)))
    D = monomial_to_dubiner(M, k)
    P = w.points[::211]
    u2 = oracle_mod.oracle_eval(V, T, M, k, w.h, P, field_mode=2)
    u0 = oracle_mod.oracle_eval(V, T, D, k, w.h, P)
    assert np.abs(u2 - u0).max() < 1e-12 * np.abs(u0).max()
