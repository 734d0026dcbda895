"""SIAC oracle -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
may import this package.  The product path (include/siac.h + the CUDA library in
paper_conf_sc_0007k13_b200/csrc) shares no code, tables or headers with it.

Contents
  kernel_coefficients(k)  exact rational c_gamma of the SIAC kernel
  bspline_moments(k, l)   exact moments of the centred B-spline of order k+1
  oracle_eval(...)        u*(x) by the plain definition, Eq. (1) (L213-235), integrated
                          exactly per Eq. (2) (L256-280) -- C core in siac_oracle.c
  kernel_values, bspline_values, dubiner_values
                          the C core's building blocks, exported for the pins in tests/

Parity pins (tests/test_oracle_*.py) tie every function to something other than itself:
textbook B-spline values, classical kernel coefficients, exact moments, closed-form
1D convolutions, exact-rational brute force, polynomial reproduction, the constant
field, adaptive quadrature and the superconvergence order.  No function here is
"parity unpinned".
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from fractions import Fraction

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "siac_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


_SRC3 = os.path.join(_HERE, "siac_oracle3d.c")


def build_oracle(force: bool = False) -> str:
    """Compile siac_oracle.c + siac_oracle3d.c -> oracle/liboracle.so (gcc -O2 -fopenmp)."""
    if force or not os.path.exists(_LIB) or any(os.path.getmtime(_LIB) < os.path.getmtime(f) for f in (_SRC, _SRC3)):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", _LIB, _SRC, _SRC3, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build_oracle()
        lib = ctypes.CDLL(_LIB)
        D, L, I = ctypes.POINTER(ctypes.c_double), ctypes.c_long, ctypes.c_int
        lib.oracle_siac_eval.restype = I
        lib.oracle_siac_eval.argtypes = [I, ctypes.c_double, I, D, D, L, ctypes.POINTER(ctypes.c_int), L,
                                         I, D, I, D, I, D, D, I, D, D, D, L, D, D, I, I, D, D]
        lib.oracle_kernel_many.argtypes = [I, D, D, L, D]
        lib.oracle_kernel_shifted_many.argtypes = [I, D, ctypes.c_double, D, L, D]
        lib.oracle_siac_eval3.restype = I
        lib.oracle_siac_eval3.argtypes = [I, ctypes.c_double, I, D, D, L, ctypes.POINTER(ctypes.c_int), L,
                                          I, D, I, D, I, D, D, D, L, D, D, I]
        lib.oracle_bspline_many.argtypes = [I, D, L, D]
        lib.oracle_dubiner_many.argtypes = [I, D, D, L, D]
        _lib = lib
    return _lib


def _dp(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


# ----------------------------------------------------------------------------- kernel

def bspline_moments(k: int, l: int) -> Fraction:
    """mu_l = int psi_{k+1}(t) t^l dt, exactly.

    psi_{k+1} (order k+1, centred, unit knots) is the density of U_1 + ... + U_{k+1} with
    U_i iid uniform(-1/2, 1/2) (the (k+1)-fold convolution of the unit box), so mu_l is the
    l-th moment of that sum: expand by the multinomial theorem with
    E[U^m] = (1/2)^m / (m+1) for even m and 0 for odd m."""
    def umom(m):
        return Fraction(0) if m % 2 else Fraction(1, 2 ** m * (m + 1))

    # moments of partial sums by repeated binomial convolution
    mom = [Fraction(1)] + [Fraction(0)] * l          # moments of the empty sum
    for _ in range(k + 1):
        new = []
        for n in range(l + 1):
            new.append(sum(math.comb(n, j) * mom[j] * umom(n - j) for j in range(n + 1)))
        mom = new
    return mom[l]


def kernel_coefficients(k: int) -> list[Fraction]:
    """c_gamma, gamma = 0..2k, of K(t) = sum_g c_g psi_{k+1}(t - x_g), x_g = -k + g.

    PAPER.md L196-208: r = 2k is "the upper bound on the polynomial degree that the
    B-splines are capable of reproducing through convolution", i.e. the moment conditions
        int K(t) dt = 1,   int K(t) t^m dt = 0,  m = 1..2k.
    With int psi(t - x_g) t^m dt = sum_l C(m,l) x_g^(m-l) mu_l this is a (2k+1)^2 linear
    system, solved here by exact Gaussian elimination over the rationals."""
    n = 2 * k + 1
    mu = [bspline_moments(k, l) for l in range(n)]
    xg = [Fraction(g - k) for g in range(n)]
    A = [[sum(math.comb(m, l) * xg[g] ** (m - l) * mu[l] for l in range(m + 1)) for g in range(n)]
         for m in range(n)]
    b = [Fraction(1)] + [Fraction(0)] * (n - 1)
    # Gauss-Jordan with exact pivots
    M = [row[:] + [b[i]] for i, row in enumerate(A)]
    for col in range(n):
        piv = next(r for r in range(col, n) if M[r][col] != 0)
        M[col], M[piv] = M[piv], M[col]
        pv = M[col][col]
        M[col] = [v / pv for v in M[col]]
        for r in range(n):
            if r != col and M[r][col] != 0:
                f = M[r][col]
                M[r] = [a - f * c for a, c in zip(M[r], M[col])]
    return [M[i][n] for i in range(n)]


def kernel_coefficients_shifted(k: int, lam) -> list[Fraction]:
    """The one-sided kernel of ref [21] (Ryan & Shu 2003; "an asymmetric
    (one-sided) stencil is used [21]"; reading R4): the 2k+1 B-spline nodes shifted to
    x_g = -k + g + lambda, the coefficients solving the SAME moment conditions as the symmetric
    kernel at the shifted nodes,
        int K(t) dt = 1,   int K(t) t^m dt = 0,  m = 1..2k,
    by exact Gauss-Jordan over the rationals (lambda converted exactly from its double)."""
    lam = Fraction(lam)
    n = 2 * k + 1
    mu = [bspline_moments(k, l) for l in range(n)]
    xg = [Fraction(g - k) + lam for g in range(n)]
    A = [[sum(math.comb(m, l) * xg[g] ** (m - l) * mu[l] for l in range(m + 1)) for g in range(n)]
         for m in range(n)]
    M = [row[:] + [Fraction(1 if i == 0 else 0)] for i, row in enumerate(A)]
    for col in range(n):
        piv = next(r for r in range(col, n) if M[r][col] != 0)
        M[col], M[piv] = M[piv], M[col]
        pv = M[col][col]
        M[col] = [v / pv for v in M[col]]
        for r in range(n):
            if r != col and M[r][col] != 0:
                f = M[r][col]
                M[r] = [a - f * c for a, c in zip(M[r], M[col])]
    return [M[i][n] for i in range(n)]


def onesided_shift(k: int, h: float, x, lo: float, hi: float):
    """Node shift lambda(x) of the one-sided kernel on an axis [lo, hi] (reading R4):
    the smallest |lambda| that keeps the support x + h [-(3k+1)/2 + lambda, (3k+1)/2 + lambda]
    inside [lo, hi]; 0 in the interior (the symmetric kernel)."""
    H = 0.5 * (3 * k + 1)
    x = np.asarray(x, dtype=np.float64)
    return np.maximum(0.0, H - (x - lo) / h) + np.minimum(0.0, (hi - x) / h - H)


def kernel_values_shifted(k: int, c, lam: float, t) -> np.ndarray:
    """K(t) = sum_g c_g psi(t - (g - k + lam)) from the C core (Cox-de Boor)."""
    lib = _load()
    t = np.ascontiguousarray(t, dtype=np.float64)
    c = np.ascontiguousarray([float(v) for v in c], dtype=np.float64)
    out = np.empty_like(t)
    lib.oracle_kernel_shifted_many(k, _dp(c), float(lam), _dp(t), t.size, _dp(out))
    return out


def kernel_values(k: int, t) -> np.ndarray:
    """K(t) from the C core (Cox-de Boor) with the exact coefficients rounded to double."""
    lib = _load()
    t = np.ascontiguousarray(t, dtype=np.float64)
    c = np.array([float(v) for v in kernel_coefficients(k)])
    out = np.empty_like(t)
    lib.oracle_kernel_many(k, _dp(c), _dp(t), t.size, _dp(out))
    return out


def bspline_values(k: int, t) -> np.ndarray:
    lib = _load()
    t = np.ascontiguousarray(t, dtype=np.float64)
    out = np.empty_like(t)
    lib.oracle_bspline_many(k, _dp(t), t.size, _dp(out))
    return out


def dubiner_values(k: int, xi, eta) -> np.ndarray:
    lib = _load()
    xi = np.ascontiguousarray(xi, dtype=np.float64)
    eta = np.ascontiguousarray(eta, dtype=np.float64)
    nb = (k + 1) * (k + 2) // 2
    out = np.empty((xi.size, nb))
    lib.oracle_dubiner_many(k, _dp(xi), _dp(eta), xi.size, _dp(out))
    return out


# ----------------------------------------------------------------------------- evaluation

def gl_sizes(k: int, field_mode: int = 0, field_deg: int = 0) -> tuple[int, int]:
    """Gauss-Legendre sizes (nx, ny) exact for the strip integrand.

    On a strip y2 = g(x) + (q(x) - g(x)) (1 + eta)/2 with g, q linear in x:
      dG field (degree k):      x-degree K1 k + K2 k + u k + Jacobian 1 = 3k+1, eta-degree 2k;
      monomial field y1^i y2^j (i, j <= d): x-degree 2k + 2d + 1, eta-degree k + d.
    An n-point Gauss-Legendre rule is exact to degree 2n-1."""
    if field_mode in (0, 2):
        dx, dy = 3 * k + 1, 2 * k
    else:
        dx, dy = 2 * k + 2 * field_deg + 1, k + field_deg
    return (dx + 2) // 2, (dy + 2) // 2


def oracle_eval(V, T, C, k: int, h: float, points, periodic: int = 3,
                domain=(0.0, 0.0, 1.0, 1.0), field_mode: int = 0, field_deg: int = 0,
                use_grid: bool | None = None, nthreads: int = 0, return_area: bool = False,
                boundary: int = 0):
    """u*(x) at every point (Eq. (1)); see siac_oracle.c for the method.

    V (nv,2) f64; T (nt,3) int; C: (nt, (k+1)(k+2)/2) Dubiner modes (field_mode 0), the
    (d+1)^2 coefficients a[i, j] of y1^i y2^j (field_mode 1, d = field_deg), or (field_mode 2,
    the library's SIAC_BASIS_MONOMIAL_REF) per-triangle coefficients of r^a s^b on the unit
    reference triangle (y = v0 + r (v1 - v0) + s (v2 - v0)), ordered by a + b, then b.
    boundary: 0 = zero extension on non-periodic axes; 1 = the one-sided kernel of ref [21] on
    non-periodic axes (per point: lambda by onesided_shift, coefficients by
    kernel_coefficients_shifted)."""
    lib = _load()
    V = np.ascontiguousarray(V, dtype=np.float64)
    T = np.ascontiguousarray(T, dtype=np.int32)
    C = np.ascontiguousarray(C, dtype=np.float64)
    P = np.ascontiguousarray(points, dtype=np.float64).reshape(-1, 2)
    dom = np.ascontiguousarray(domain, dtype=np.float64)
    W = (3 * k + 1) * h
    if periodic & 1 and W > dom[2] - dom[0] + 1e-12:
        raise ValueError("stencil width exceeds the periodic x-extent")
    if periodic & 2 and W > dom[3] - dom[1] + 1e-12:
        raise ValueError("stencil width exceeds the periodic y-extent")
    kc = np.array([float(v) for v in kernel_coefficients(k)])
    nx, ny = gl_sizes(k, field_mode, field_deg)
    gx, gwx = np.polynomial.legendre.leggauss(nx)
    gy, gwy = np.polynomial.legendre.leggauss(ny)
    out = np.zeros(len(P))
    area = np.zeros(len(P)) if return_area else None
    pt_lam = pt_coef = None
    if boundary == 1 and periodic != 3:
        if (not periodic & 1 and W > dom[2] - dom[0] + 1e-12) or (not periodic & 2 and W > dom[3] - dom[1] + 1e-12):
            raise ValueError("one-sided kernel: stencil width exceeds the domain")
        pt_lam = np.zeros((len(P), 2))
        for ax in (0, 1):
            if not periodic & (1 << ax):
                pt_lam[:, ax] = onesided_shift(k, h, P[:, ax], dom[ax], dom[ax + 2])
        cache = {}
        pt_coef = np.empty((len(P), 2, 2 * k + 1))
        for i in range(len(P)):
            for ax in (0, 1):
                lv = float(pt_lam[i, ax])
                if lv not in cache:
                    cache[lv] = np.array([float(v) for v in kernel_coefficients_shifted(k, lv)])
                pt_coef[i, ax] = cache[lv]
        pt_lam = np.ascontiguousarray(pt_lam)
        pt_coef = np.ascontiguousarray(pt_coef)
    if use_grid is None:
        use_grid = len(T) > 2000
    rc = lib.oracle_siac_eval(k, float(h), int(periodic), _dp(dom), _dp(V), len(V),
                              T.ctypes.data_as(ctypes.POINTER(ctypes.c_int)), len(T),
                              int(field_mode), _dp(C), int(field_deg), _dp(kc),
                              nx, _dp(gx), _dp(gwx), ny, _dp(gy), _dp(gwy),
                              _dp(P), len(P), _dp(out),
                              _dp(area) if return_area else None, int(bool(use_grid)), int(nthreads),
                              _dp(pt_lam) if pt_lam is not None else None,
                              _dp(pt_coef) if pt_coef is not None else None)
    if rc != 0:
        raise RuntimeError(f"oracle_siac_eval failed ({rc})")
    return (out, area) if return_area else out


def omp_threads() -> int:
    """Threads the C core will use by default (OpenMP default = all host cores available)."""
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


# ----------------------------------------------------------------------------- 3D (NEXT-4)

def n_modes3(k: int) -> int:
    return (k + 1) * (k + 2) * (k + 3) // 6


def oracle_eval3(V, T, C, k: int, h: float, points, periodic: int = 7,
                 domain=(0.0, 0.0, 0.0, 1.0, 1.0, 1.0), field_mode: int = 0, field_deg: int = 0,
                 nthreads: int = 0, return_volume: bool = False):
    """u*(x) on a tetrahedral mesh (the 3D form of Eq. (1); siac_oracle3d.c for the method).

    V (nv,3); T (nt,4) int; C: (nt, n_modes3(k)) coefficients of r^a s^b t^c on the unit
    reference tetrahedron (y = v0 + r (v1-v0) + s (v2-v0) + t (v3-v0); modes by n = a+b+c, then
    c, then b) for field_mode 0, or (d+1)^3 coefficients a[i, j, l] of y1^i y2^j y3^l
    (field_mode 1, d = field_deg).  periodic: bit d = axis d."""
    lib = _load()
    V = np.ascontiguousarray(V, dtype=np.float64)
    T = np.ascontiguousarray(T, dtype=np.int32)
    C = np.ascontiguousarray(C, dtype=np.float64)
    P = np.ascontiguousarray(points, dtype=np.float64).reshape(-1, 3)
    dom = np.ascontiguousarray(domain, dtype=np.float64)
    W = (3 * k + 1) * h
    for d in range(3):
        if periodic & (1 << d) and W > dom[d + 3] - dom[d] + 1e-12:
            raise ValueError("stencil width exceeds a periodic extent")
    kc = np.array([float(v) for v in kernel_coefficients(k)])
    # degree of the x-integrand K(x) S(x) between breakpoints: K_x (k) times the section integral
    # of K_y K_z u (total degree 2k + k for dG, 2k + 3d for x^i y^j z^l) over a polygon whose
    # vertices move linearly in x (+2); the y- and z-integrands have lower degree.  An n-point
    # Gauss rule is exact to degree 2n-1.
    deg = (k + 3 * k if field_mode == 0 else 3 * k + 3 * field_deg) + 2
    n = deg // 2 + 1
    g, w = np.polynomial.legendre.leggauss(n)
    out = np.zeros(len(P))
    vol = np.zeros(len(P)) if return_volume else None
    rc = lib.oracle_siac_eval3(k, float(h), int(periodic), _dp(dom), _dp(V), len(V),
                               T.ctypes.data_as(ctypes.POINTER(ctypes.c_int)), len(T), int(field_mode), _dp(C),
                               int(field_deg), _dp(kc), n, _dp(g), _dp(w), _dp(P), len(P), _dp(out),
                               _dp(vol) if return_volume else None, int(nthreads))
    if rc != 0:
        raise RuntimeError(f"oracle_siac_eval3 failed ({rc})")
    return (out, vol) if return_volume else out
