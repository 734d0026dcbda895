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
