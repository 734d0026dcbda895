"""Pins for the 3D oracle and the 3D input generators.

What fixes the expected values (none of it re-types the oracle):
  * u = 1 -> u* = 1 and the integrated volume is the stencil volume W^3 (the kernel integrates
    to 1, L202-205; the pieces partition the stencil);
  * x^a y^b z^c with a, b, c <= 2k is reproduced, and degree 2k+2 picks up exactly
    m_{2k+2} h^{2k+2} per axis (the closed form of the tensor-product convolution);
  * a global polynomial of degree k given as per-tetrahedron reference monomials is reproduced;
  * separable lift on the structured Kuhn mesh: u_h = f(x) piecewise polynomial per cell column
    gives u*(x, y, z) = (K_h * f)(x), the exact-rational 1D routine of test_oracle_pins (itself
    pinned to SURVEY A4's exact values) -- this exercises the cuts of the tetrahedra's diagonal
    faces by every kernel plane;
  * superconvergence order >= 2k+1 - 0.2 on sin(2 pi x) sin(2 pi y) sin(2 pi z) (k = 1);
  * the input generators: Kuhn meshes tile the cube, the L2 projection reproduces polynomials.
"""
import math
from fractions import Fraction as Fr

import numpy as np
import pytest

from paper_conf_sc_0007k13_b200.inputs import mesh3d as m3

from test_oracle_pins import LEG, MODES_1D, _gold_1d, _moment, exact_1d


def _vol(V, T):
    a, b, c = V[T[:, 1]] - V[T[:, 0]], V[T[:, 2]] - V[T[:, 0]], V[T[:, 3]] - V[T[:, 0]]
    return np.einsum("ij,ij->i", a, np.cross(b, c)) / 6.0


def test_generators():
    V, T = m3.structured_mesh3(3)
    v = _vol(V, T)
    assert np.all(v > 0) and abs(v.sum() - 1.0) < 1e-14 and len(T) == 6 * 27
    V, T = m3.lattice_delaunay_mesh3(2000, seed=1)
    v = _vol(V, T)
    assert np.all(v > 0) and abs(v.sum() - 1.0) < 1e-12
    f = lambda x, y, z: 0.5 - x * y + 2 * z * z * x  # noqa: E731
    C = m3.project3(V, T, 3, f)
    P = m3.eval_points3(V, T)[:: 97]
    ti = np.arange(0, len(P) * 97, 97) // 4
    # evaluate the modes at the points: r s t from the affine map
    v0, v1, v2, v3 = (V[T[ti, i]] for i in range(4))
    A = np.stack([v1 - v0, v2 - v0, v3 - v0], axis=2)
    rst = np.linalg.solve(A, (P - v0)[..., None])[..., 0]
    phi = np.stack([rst[:, 0] ** a * rst[:, 1] ** b * rst[:, 2] ** c for a, b, c in m3.mode_list3(3)], axis=1)
    assert np.abs((phi * C[ti]).sum(1) - f(P[:, 0], P[:, 1], P[:, 2])).max() < 1e-12


@pytest.mark.parametrize("k,mesh", [(1, "s"), (2, "s"), (3, "s"), (1, "d")])
def test_constant_field_and_volume(oracle_mod, k, mesh):
    if mesh == "s":
        V, T = m3.structured_mesh3(3 if k == 3 else 4)
        h = 0.1 if k == 3 else 0.07
    else:
        V, T = m3.lattice_delaunay_mesh3(1500, seed=2)
        h = 0.08
    C = np.zeros((len(T), m3.n_modes3(k)))
    C[:, 0] = 1.0
    P = np.random.default_rng(k).uniform(-0.1, 1.1, (4, 3))
    P[0] = [0, 0, 0]
    u, vol = oracle_mod.oracle_eval3(V, T, C, k, h, P, return_volume=True)
    assert np.abs(u - 1).max() < 1e-13
    assert np.abs(vol - ((3 * k + 1) * h) ** 3).max() < 1e-14


@pytest.mark.parametrize("k", [1, 2])
def test_monomial_reproduction_and_negative_control(oracle_mod, k):
    V, T = m3.lattice_delaunay_mesh3(700, seed=4)
    h = 0.035 if k == 2 else 0.05
    W = (3 * k + 1) * h
    P = np.random.default_rng(5).uniform(W / 2 + 0.01, 1 - W / 2 - 0.01, (3 if k == 1 else 2, 3))
    d = 2 * k + 2
    cases = [(2 * k, 0, 1), (0, 2 * k, 2 * k), (d, 0, 0)] if k == 1 else [(2 * k, 1, 0), (d, 0, 0)]
    for a, b, c in cases:
        fd = max(a, b, c)                  # the field's per-variable degree (sets the rule size)
        A = np.zeros((fd + 1, fd + 1, fd + 1))
        A[a, b, c] = 1.0
        u = oracle_mod.oracle_eval3(V, T, A, k, h, P, periodic=0, field_mode=1, field_deg=fd)

        def conv(x, n):
            return sum(math.comb(n, l) * x ** (n - l) * h ** l * float(_moment(k, l)) for l in range(n + 1))

        expect = np.array([conv(x[0], a) * conv(x[1], b) * conv(x[2], c) for x in P])
        assert np.abs(u - expect).max() < 1e-13, (a, b, c)
        exact = P[:, 0] ** a * P[:, 1] ** b * P[:, 2] ** c
        if max(a, b, c) <= 2 * k:
            assert np.abs(u - exact).max() < 1e-13
        else:
            assert np.abs(u - exact).max() > 1e-3 * h ** d


@pytest.mark.parametrize("k", [1, 2])
def test_dg_polynomial_reproduction(oracle_mod, k):
    V, T = m3.lattice_delaunay_mesh3(1500, seed=6)
    f = lambda x, y, z: 0.3 + (x - 0.2 * y + 0.1 * z) ** k - 0.5 * x * y ** (k - 1)  # noqa: E731
    C = m3.project3(V, T, k, f)
    h = 0.05 if k == 2 else 0.07
    W = (3 * k + 1) * h
    P = np.random.default_rng(7).uniform(W / 2 + 0.01, 1 - W / 2 - 0.01, (3, 3))
    u = oracle_mod.oracle_eval3(V, T, C, k, h, P, periodic=0)
    assert np.abs(u - f(P[:, 0], P[:, 1], P[:, 2])).max() < 1e-13


@pytest.mark.parametrize("k", [1, 2])
def test_separable_lift_3d(oracle_mod, k):
    """u_h(x, y, z) = f(x) on the periodic N^3 Kuhn mesh -> u* = f*(x) for all (y, z)."""
    N = {1: 4, 2: 8}[k]
    modes = MODES_1D[k]
    V, T = m3.structured_mesh3(N)

    def f(X, Y, Z):
        i = np.clip(np.floor(X * N).astype(int), 0, N - 1)
        xi = 2 * (X - (i + 0.5) / N) * N
        out = np.zeros_like(X)
        for j in range(k + 1):
            amp = np.array([float(modes[ii][j]) for ii in range(N)])[i]
            out += amp * np.polynomial.legendre.legval(xi, [0] * j + [1])
        return out

    C = m3.project3(V, T, k, f)
    xs = [x for kk, NN, x, _ in _gold_1d() if kk == k][:2]
    yz = [(0.0, 0.0), (0.3, 0.71)]
    P = np.array([[float(x), y, z] for x in xs for y, z in yz])
    u = oracle_mod.oracle_eval3(V, T, C, k, 1 / N, P)
    expect = np.array([float(exact_1d(k, N, modes, x)) for x in xs for _ in yz])
    assert np.abs(u - expect).max() < 1e-13


def test_superconvergence_k1(oracle_mod):
    """Filtered error at element points decays at order >= 2k+1 - 0.2 (k = 1: 3; L2-projected
    input, expected 2k+2 = 4) on sin sin sin, structured periodic Kuhn meshes, h = 1/N."""
    errs = []
    rng = np.random.default_rng(11)
    Ns = (4, 8, 16)
    for N in Ns:
        V, T = m3.structured_mesh3(N)
        C = m3.project3(V, T, 1, m3.sin3)
        sel = rng.choice(len(T), size=min(len(T), 6), replace=False)
        P = m3.eval_points3(V, T[sel])
        u = oracle_mod.oracle_eval3(V, T, C, 1, 1 / N, P)
        errs.append(np.abs(u - m3.sin3(P[:, 0], P[:, 1], P[:, 2])).max())
    rates = [math.log(errs[i] / errs[i + 1]) / math.log(Ns[i + 1] / Ns[i]) for i in range(len(errs) - 1)]
    assert min(rates) >= 2.8, (errs, rates)
