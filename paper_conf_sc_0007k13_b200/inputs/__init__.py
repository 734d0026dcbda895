"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module generates INPUTS only: meshes, evaluation points and dG modal coefficients.
It holds none of the SIAC method's arithmetic (no kernel, no clipping, no convolution);
both the oracle (oracle/) and the CUDA path (csrc/) consume what it produces.

Workload recipe:
  * structured (config 1): N x N squares of [0,1]^2, each split by the "/" diagonal
    (Fig. 2(a));
  * unstructured (configs 2, 4, 5): Delaunay triangulation ("2D
    unstructured triangular meshes created using Delaunay triangulation") of a jittered
    triangular lattice with equally spaced, periodically matched boundary nodes;
  * graded (config 3, the paper's "highly varying element sizes", L712-713): the same
    lattice mapped per axis by phi(u) = u - 0.6 sin(2 pi u)/(2 pi) before triangulating;
  * field: u = sin(2 pi x) sin(2 pi y) L2-projected per element onto the orthonormal
    Dubiner basis of P_k (paper L716-718: 3/6/10 modes for P1/P2/P3);
  * points: nodes of the symmetric degree-2k triangle rule in every element
    ("the evaluation points are the quadrature points").
Every generator takes an explicit seed; nothing depends on global RNG state.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

from .eval_rules import EVAL_RULES

__all__ = [
    "Workload", "structured_mesh", "lattice_delaunay_mesh", "eval_points",
    "dubiner_eval", "project", "random_modes", "make_config", "CONFIGS",
    "n_modes", "max_edge", "triangle_areas",
]


def n_modes(k: int) -> int:
    """Number of P_k modes on a triangle: (k+1)(k+2)/2."""
    return (k + 1) * (k + 2) // 2


# ----------------------------------------------------------------------------- meshes

def structured_mesh(n: int, x0=0.0, y0=0.0, lx=1.0, ly=1.0):
    """N x N squares split by the '/' diagonal -> (vertices (nv,2) f64, triangles (nt,3) i32).

    Square (i, j) with corners v00, v10, v11, v01 gives triangles (v00, v10, v11) and
    (v00, v11, v01), both counter-clockwise."""
    xs = x0 + lx * np.arange(n + 1) / n
    ys = y0 + ly * np.arange(n + 1) / n
    X, Y = np.meshgrid(xs, ys, indexing="xy")
    V = np.stack([X.ravel(), Y.ravel()], axis=1).astype(np.float64)
    idx = lambda i, j: j * (n + 1) + i  # noqa: E731
    tris = []
    for j in range(n):
        for i in range(n):
            v00, v10, v11, v01 = idx(i, j), idx(i + 1, j), idx(i + 1, j + 1), idx(i, j + 1)
            tris.append((v00, v10, v11))
            tris.append((v00, v11, v01))
    return V, np.asarray(tris, dtype=np.int32)


def _grading_map(u):
    return u - 0.6 * np.sin(2 * np.pi * u) / (2 * np.pi)


def lattice_delaunay_mesh(ntri_target: int, seed: int, graded: bool = False, jitter: float = 0.45):
    """Delaunay mesh of a jittered triangular lattice on [0,1]^2 with ~ntri_target triangles.

    Boundary nodes are equally spaced and identical on opposite sides (periodic-compatible).
    Interior nodes: rows spaced sqrt(3)/2 dx, odd rows offset dx/2, uniform jitter
    +-jitter*(dx, dy), kept >= 0.1 dx (0.1 dy) away from the boundary."""
    from scipy.spatial import Delaunay

    rng = np.random.default_rng(seed)
    # a Delaunay triangulation of a convex domain with N nodes, B on the hull, has 2N-B-2 triangles
    nnodes = ntri_target / 2.0
    dx = math.sqrt(2.0 / (math.sqrt(3.0) * nnodes))
    nx = max(2, int(round(1.0 / dx)))
    ny = max(2, int(round(1.0 / (dx * math.sqrt(3.0) / 2.0))))
    dx, dy = 1.0 / nx, 1.0 / ny
    pts = []
    for j in range(1, ny):
        off = 0.5 if (j % 2) else 0.0
        i0 = 0 if off else 1
        xs = (np.arange(i0, nx) + off) * dx
        ys = np.full_like(xs, j * dy)
        pts.append(np.stack([xs, ys], axis=1))
    P = np.concatenate(pts, axis=0)
    P = P + rng.uniform(-jitter, jitter, size=P.shape) * np.array([dx, dy])
    P[:, 0] = np.clip(P[:, 0], 0.1 * dx, 1.0 - 0.1 * dx)
    P[:, 1] = np.clip(P[:, 1], 0.1 * dy, 1.0 - 0.1 * dy)
    bx = np.arange(nx + 1) * dx
    by = np.arange(1, ny) * dy
    bx[-1] = 1.0
    B = np.concatenate([
        np.stack([bx, np.zeros_like(bx)], 1), np.stack([bx, np.ones_like(bx)], 1),
        np.stack([np.zeros_like(by), by], 1), np.stack([np.ones_like(by), by], 1),
    ])
    V = np.concatenate([B, P], axis=0)
    if graded:
        V = _grading_map(V)
        V[np.abs(V) < 1e-15] = 0.0
        V[np.abs(V - 1.0) < 1e-15] = 1.0
    tri = Delaunay(V)
    T = tri.simplices.astype(np.int64)
    a = V[T[:, 1]] - V[T[:, 0]]
    b = V[T[:, 2]] - V[T[:, 0]]
    det = a[:, 0] * b[:, 1] - a[:, 1] * b[:, 0]
    keep = np.abs(det) > 1e-10 * np.abs(det).mean()
    T, det = T[keep], det[keep]
    neg = det < 0
    T[neg] = T[neg][:, [0, 2, 1]]
    # drop unreferenced vertices and renumber
    used = np.unique(T)
    remap = -np.ones(len(V), dtype=np.int64)
    remap[used] = np.arange(len(used))
    return V[used].astype(np.float64), remap[T].astype(np.int32)


def triangle_areas(V, T):
    a = V[T[:, 1]] - V[T[:, 0]]
    b = V[T[:, 2]] - V[T[:, 0]]
    return 0.5 * np.abs(a[:, 0] * b[:, 1] - a[:, 1] * b[:, 0])


def max_edge(V, T) -> float:
    e = [np.linalg.norm(V[T[:, (i + 1) % 3]] - V[T[:, i]], axis=1) for i in range(3)]
    return float(np.max(np.stack(e)))


# ----------------------------------------------------------------------------- points

def eval_points(V, T, k: int) -> np.ndarray:
    """Nodes of the degree-2k symmetric rule mapped into every element, element-major.

    Point = v0 + r (v1 - v0) + s (v2 - v0) for each rule node (r, s)."""
    rule = np.asarray(EVAL_RULES[k], dtype=np.float64)
    r, s = rule[:, 0], rule[:, 1]
    v0, v1, v2 = V[T[:, 0]], V[T[:, 1]], V[T[:, 2]]
    P = (v0[:, None, :] + r[None, :, None] * (v1 - v0)[:, None, :]
         + s[None, :, None] * (v2 - v0)[:, None, :])
    return np.ascontiguousarray(P.reshape(-1, 2))


# ----------------------------------------------------------------------------- dG field

def _mode_list(k):
    """(p, q) in the order used everywhere: total degree n = p+q ascending, then q ascending."""
    return [(n - q, q) for n in range(k + 1) for q in range(n + 1)]


def dubiner_eval(k: int, xi: np.ndarray, eta: np.ndarray) -> np.ndarray:
    """Orthonormal Dubiner modes on {xi, eta >= -1, xi + eta <= 0} -> (len(xi), n_modes).

    phi_pq = sqrt((2p+1)(p+q+1)/2) P_p(a) ((1-b)/2)^p P_q^(2p+1,0)(b),
    a = 2(1+xi)/(1-eta) - 1, b = eta (SURVEY §8(b) basis convention; Q8).
    Evaluated with scipy's Jacobi polynomials at points with eta < 1."""
    from scipy.special import eval_jacobi, eval_legendre

    xi = np.asarray(xi, dtype=np.float64)
    eta = np.asarray(eta, dtype=np.float64)
    a = 2.0 * (1.0 + xi) / (1.0 - eta) - 1.0
    out = []
    for (p, q) in _mode_list(k):
        c = math.sqrt((2 * p + 1) * (p + q + 1) / 2.0)
        out.append(c * eval_legendre(p, a) * ((1.0 - eta) / 2.0) ** p * eval_jacobi(q, 2 * p + 1, 0, eta))
    return np.stack(out, axis=-1)


def _ref_rule(n: int):
    """Collapsed (Duffy) Gauss-Legendre rule on the reference triangle: nodes (xi, eta), weights.

    Exact for polynomials of total degree <= 2n-2 on the triangle (area 2)."""
    g, w = np.polynomial.legendre.leggauss(n)
    A, Bn = np.meshgrid(g, g, indexing="ij")
    WA, WB = np.meshgrid(w, w, indexing="ij")
    xi = (1.0 + A) * (1.0 - Bn) / 2.0 - 1.0
    eta = Bn
    W = WA * WB * (1.0 - Bn) / 2.0
    return xi.ravel(), eta.ravel(), W.ravel()


def project(V, T, k: int, f, n_quad: int = 10, chunk: int = 1 << 17) -> np.ndarray:
    """L2 projection of f(x, y) (vectorised callable) onto P_k on every triangle.

    With the orthonormal basis the element mass matrix is (|T|/2) I, so
    c_i = integral over the reference triangle of f(y(xi, eta)) phi_i(xi, eta)."""
    xi, eta, W = _ref_rule(n_quad)
    Phi = dubiner_eval(k, xi, eta)                      # (nq, nb)
    r, s = (xi + 1.0) / 2.0, (eta + 1.0) / 2.0
    out = np.empty((len(T), n_modes(k)), dtype=np.float64)
    for c0 in range(0, len(T), chunk):
        Tc = T[c0:c0 + chunk]
        v0, v1, v2 = V[Tc[:, 0]], V[Tc[:, 1]], V[Tc[:, 2]]
        X = v0[:, None, 0] + r[None, :] * (v1 - v0)[:, None, 0] + s[None, :] * (v2 - v0)[:, None, 0]
        Y = v0[:, None, 1] + r[None, :] * (v1 - v0)[:, None, 1] + s[None, :] * (v2 - v0)[:, None, 1]
        F = f(X, Y)                                     # (nt, nq)
        out[c0:c0 + chunk] = (F * W[None, :]) @ Phi
    return out


def sinsin(x, y):
    return np.sin(2 * np.pi * x) * np.sin(2 * np.pi * y)


def random_modes(nt: int, k: int, seed: int) -> np.ndarray:
    """Seeded uniform(-1, 1) modal coefficients (a field with no structure, for parity tests)."""
    return np.random.default_rng(seed).uniform(-1.0, 1.0, size=(nt, n_modes(k)))


# ----------------------------------------------------------------------------- configs

@dataclass
class Workload:
    name: str
    k: int
    h: float
    V: np.ndarray
    T: np.ndarray
    C: np.ndarray
    points: np.ndarray
    periodic: int = 3
    domain: tuple = (0.0, 0.0, 1.0, 1.0)
    seed: int = 0
    meta: dict = field(default_factory=dict)

    @property
    def n_points(self):
        return len(self.points)


CONFIGS = {
    1: dict(kind="structured", n=20, k=1, desc="structured 20x20 (800 tris), P1, h=1/20, 3 pts/elt"),
    2: dict(kind="delaunay", ntri=4096, k=2, desc="Delaunay ~4K tris, P2, h=max edge, 6 pts/elt"),
    3: dict(kind="graded", ntri=16384, k=3, desc="graded Delaunay ~16K tris, P3, h=max edge, 12 pts/elt"),
    4: dict(kind="delaunay", ntri=65536, k=4, desc="Delaunay ~65K tris, P4, h=max edge, 16 pts/elt"),
    5: dict(kind="delaunay", ntri=1048576, k=3, desc="Delaunay ~1M tris, P3, h=max edge, 12 pts/elt"),
}


def make_config(cfg: int, field_kind: str = "sinsin", seed: int | None = None) -> Workload:
    """Build BASELINE.json config `cfg` (1..5) with seed 1000+cfg."""
    spec = CONFIGS[cfg]
    seed = 1000 + cfg if seed is None else seed
    k = spec["k"]
    if spec["kind"] == "structured":
        V, T = structured_mesh(spec["n"])
        h = 1.0 / spec["n"]
    else:
        V, T = lattice_delaunay_mesh(spec["ntri"], seed, graded=(spec["kind"] == "graded"))
        h = max_edge(V, T)
    if field_kind == "sinsin":
        C = project(V, T, k, sinsin, n_quad=k + 6)
    else:
        C = random_modes(len(T), k, seed + 7)
    P = eval_points(V, T, k)
    return Workload(name=f"cfg{cfg}", k=k, h=h, V=V, T=T, C=C, points=P, seed=seed,
                    meta=dict(desc=spec["desc"], ntri=len(T), npts=len(P)))
