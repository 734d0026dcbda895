"""Seeded synthetic 3D inputs: tetrahedral meshes of
the unit cube, evaluation points, and modal coefficients.  INPUTS ONLY -- no SIAC arithmetic
(no kernel, no clipping, no convolution); the 3D oracle and the CUDA path both consume them.

Recipe:
  * structured: N^3 cubes, each split into 6 tetrahedra along its main diagonal (the Kuhn /
    Freudenthal subdivision: one tetrahedron per axis permutation), conforming and
    periodic-compatible;
  * unstructured: Delaunay triangulation (scipy / Qhull) of a jittered cubic lattice plus equally
    spaced nodes on the faces of the cube matched on opposite faces (periodic-compatible),
    slivers (relative volume < 1e-6 of the mean) dropped;
  * field: per-tetrahedron coefficients of the monomials r^a s^b t^c of the unit reference
    tetrahedron (point = v0 + r (v1-v0) + s (v2-v0) + t (v3-v0)), ordered by n = a+b+c, then c,
    then b -- the library's SIAC_BASIS_MONOMIAL_REF in 3D; L2 projections of an analytic field
    or seeded random modes;
  * points: the 4 nodes of the degree-2 symmetric tetrahedron rule in every element.
"""
from __future__ import annotations

import itertools
import math

import numpy as np


def n_modes3(k: int) -> int:
    return (k + 1) * (k + 2) * (k + 3) // 6


def mode_list3(k: int):
    """(a, b, c) exponents of r, s, t in the library's order: n = a+b+c, then c, then b."""
    return [(n - b - c, b, c) for n in range(k + 1) for c in range(n + 1) for b in range(n - c + 1)]


def _orient(V, T):
    a, b, c = V[T[:, 1]] - V[T[:, 0]], V[T[:, 2]] - V[T[:, 0]], V[T[:, 3]] - V[T[:, 0]]
    det = np.einsum("ij,ij->i", a, np.cross(b, c))
    T = T.copy()
    neg = det < 0
    T[neg] = T[neg][:, [0, 2, 1, 3]]
    return T, np.abs(det)


def structured_mesh3(n: int):
    """N^3 cubes of [0,1]^3, 6 tetrahedra each (Kuhn subdivision), positively oriented."""
    g = np.arange(n + 1) / n
    X, Y, Z = np.meshgrid(g, g, g, indexing="ij")
    V = np.stack([X.ravel(), Y.ravel(), Z.ravel()], axis=1)
    idx = lambda i, j, l: (i * (n + 1) + j) * (n + 1) + l  # noqa: E731
    tets = []
    for i in range(n):
        for j in range(n):
            for l in range(n):
                for perm in itertools.permutations(range(3)):
                    p = [i, j, l]
                    path = [idx(*p)]
                    for ax in perm:
                        p[ax] += 1
                        path.append(idx(*p))
                    tets.append(path)
    T, _ = _orient(V, np.asarray(tets, dtype=np.int64))
    return V.astype(np.float64), T.astype(np.int32)


def lattice_delaunay_mesh3(ntet_target: int, seed: int, jitter: float = 0.35):
    """Delaunay mesh of a jittered cubic lattice on [0,1]^3 with about ntet_target tetrahedra
    (~5.4 tetrahedra per interior node); face nodes equally spaced and matched on opposite faces."""
    from scipy.spatial import Delaunay

    rng = np.random.default_rng(seed)
    m = max(2, int(round((ntet_target / 5.4) ** (1.0 / 3.0))))
    d = 1.0 / m
    g = np.arange(m + 1) * d
    X, Y, Z = np.meshgrid(g, g, g, indexing="ij")
    P = np.stack([X.ravel(), Y.ravel(), Z.ravel()], axis=1)
    onb = np.any((P < 1e-12) | (P > 1 - 1e-12), axis=1)
    inner = P[~onb] + rng.uniform(-jitter, jitter, size=(np.count_nonzero(~onb), 3)) * d
    inner = np.clip(inner, 0.1 * d, 1 - 0.1 * d)
    V = np.concatenate([P[onb], inner], axis=0)
    T = Delaunay(V).simplices.astype(np.int64)
    T, vol = _orient(V, T)
    keep = vol > 1e-6 * vol.mean()
    T = T[keep]
    used = np.unique(T)
    remap = -np.ones(len(V), dtype=np.int64)
    remap[used] = np.arange(len(used))
    return V[used].astype(np.float64), remap[T].astype(np.int32)


def max_edge3(V, T) -> float:
    E = [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)]
    return float(max(np.linalg.norm(V[T[:, b]] - V[T[:, a]], axis=1).max() for a, b in E))


def max_extent3(V, T) -> float:
    P = V[T]
    return float((P.max(axis=1) - P.min(axis=1)).max())


EVAL_RULE3 = np.array([[0.5854101966249685, 0.1381966011250105, 0.1381966011250105, 0.1381966011250105],
                       [0.1381966011250105, 0.5854101966249685, 0.1381966011250105, 0.1381966011250105],
                       [0.1381966011250105, 0.1381966011250105, 0.5854101966249685, 0.1381966011250105],
                       [0.1381966011250105, 0.1381966011250105, 0.1381966011250105, 0.5854101966249685]])


def eval_points3(V, T) -> np.ndarray:
    """The 4 nodes (barycentric (a, b, b, b) and permutations) of the degree-2 tetrahedron rule
    in every element, element-major -> (4 nt, 3)."""
    P = np.einsum("qv,tvd->tqd", EVAL_RULE3, V[T])
    return np.ascontiguousarray(P.reshape(-1, 3))


def _ref_rule3(n: int):
    """Collapsed Gauss-Legendre (Duffy) rule on the unit reference tetrahedron: (r, s, t), w
    (weights sum to 1/6); exact for total degree <= 2n - 3."""
    g, w = np.polynomial.legendre.leggauss(n)
    u = 0.5 * (g + 1.0)
    wu = 0.5 * w
    A, B, C = np.meshgrid(u, u, u, indexing="ij")
    WA, WB, WC = np.meshgrid(wu, wu, wu, indexing="ij")
    r = A * (1 - B) * (1 - C)
    s = B * (1 - C)
    t = C
    W = WA * WB * WC * (1 - B) * (1 - C) ** 2
    return r.ravel(), s.ravel(), t.ravel(), W.ravel()


def project3(V, T, k: int, f, n_quad: int | None = None) -> np.ndarray:
    """L2 projection of f(x, y, z) onto P_k on every tetrahedron, in the reference-monomial basis:
    c = M^{-1} b with M_ij = int_ref phi_i phi_j and b_i = int_ref phi_i f(y(r,s,t))."""
    r, s, t, W = _ref_rule3(n_quad or k + 6)
    Phi = np.stack([r ** a * s ** b * t ** c for a, b, c in mode_list3(k)], axis=1)    # (nq, nb)
    M = Phi.T @ (W[:, None] * Phi)
    v0, v1, v2, v3 = (V[T[:, i]] for i in range(4))
    X = (v0[:, None, :] + r[None, :, None] * (v1 - v0)[:, None, :] + s[None, :, None] * (v2 - v0)[:, None, :]
         + t[None, :, None] * (v3 - v0)[:, None, :])
    F = f(X[..., 0], X[..., 1], X[..., 2])                                          # (nt, nq)
    rhs = (F * W[None, :]) @ Phi
    return np.linalg.solve(M, rhs.T).T


def sin3(x, y, z):
    return np.sin(2 * np.pi * x) * np.sin(2 * np.pi * y) * np.sin(2 * np.pi * z)


def random_modes3(nt: int, k: int, seed: int) -> np.ndarray:
    return np.random.default_rng(seed).uniform(-1.0, 1.0, size=(nt, n_modes3(k)))
