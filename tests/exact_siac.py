"""Exact-rational brute-force SIAC evaluation (test helper; pure Python Fractions).

An independent third implementation used only to pin the oracle (pin P7):
  * K on each kernel cell from the truncated-power form of the centred B-spline
        psi_{k+1}(t) = (1/k!) sum_{j=0}^{k+1} (-1)^j C(k+1, j) (t + (k+1)/2 - j)_+^k
    (a textbook identity; the oracle uses Cox-de Boor instead);
  * exact Sutherland-Hodgman clipping (Alg. 1) of every periodic
    triangle image against every kernel cell, fan triangulation (L248-249);
  * exact integration of the polynomial integrand over each sub-triangle via
        int_{unit triangle} r^a s^b = a! b! / (a+b+2)!.
The field is given per triangle as a rational polynomial in PHYSICAL coordinates
{(a, b): coeff} of y1^a y2^b (evaluated at y - s for image shift s).
Cost grows fast; use only on tiny meshes.
"""
from __future__ import annotations

import math
from fractions import Fraction as Fr


# ---------------------------------------------------------------- polynomials {(a,b): Fr}

def padd(p, q):
    r = dict(p)
    for m, c in q.items():
        r[m] = r.get(m, 0) + c
    return {m: c for m, c in r.items() if c != 0}


def pmul(p, q):
    r = {}
    for (a1, b1), c1 in p.items():
        for (a2, b2), c2 in q.items():
            m = (a1 + a2, b1 + b2)
            r[m] = r.get(m, 0) + c1 * c2
    return {m: c for m, c in r.items() if c != 0}


def ppow(p, n):
    r = {(0, 0): Fr(1)}
    for _ in range(n):
        r = pmul(r, p)
    return r


def compose_affine(p, X, Y):
    """p(X(r,s), Y(r,s)) where X, Y are polynomials in (r, s)."""
    out = {}
    maxa = max((a for a, _ in p), default=0)
    maxb = max((b for _, b in p), default=0)
    Xp = [ppow(X, i) for i in range(maxa + 1)]
    Yp = [ppow(Y, i) for i in range(maxb + 1)]
    for (a, b), c in p.items():
        out = padd(out, {m: c * v for m, v in pmul(Xp[a], Yp[b]).items()})
    return out


# ---------------------------------------------------------------- kernel pieces

def kernel_cell_polys(k, coeffs):
    """[poly_i(t)] for cells i = 0..3k, cell i = [t_i, t_{i+1}], t_i = -(3k+1)/2 + i.

    Each poly is a list of Fraction coefficients in powers of t."""
    half = Fr(k + 1, 2)
    out = []
    for i in range(3 * k + 1):
        ti = Fr(-(3 * k + 1), 2) + i
        poly = [Fr(0)] * (k + 1)
        for g, cg in enumerate(coeffs):
            xg = Fr(g - k)
            for j in range(k + 2):
                a = xg - half + j                 # knot of this truncated power
                if a <= ti:                       # (t - a)_+^k is (t - a)^k on the whole cell
                    w = cg * (-1) ** j * math.comb(k + 1, j) / math.factorial(k)
                    for m in range(k + 1):        # (t - a)^k = sum_m C(k,m) t^m (-a)^(k-m)
                        poly[m] += w * math.comb(k, m) * (-a) ** (k - m)
        out.append(poly)
    return out


# ---------------------------------------------------------------- clipping

def clip(poly, inside, inter):
    """One Sutherland-Hodgman pass (Alg. 1) against one clip edge."""
    out = []
    if not poly:
        return out
    S = poly[-1]
    for E in poly:
        if inside(E):
            if not inside(S):
                out.append(inter(S, E))
            out.append(E)
        elif inside(S):
            out.append(inter(S, E))
        S = E
    return out


def clip_rect(poly, x0, x1, y0, y1):
    def ix(X):
        return lambda S, E: (X, S[1] + (X - S[0]) / (E[0] - S[0]) * (E[1] - S[1]))

    def iy(Y):
        return lambda S, E: (S[0] + (Y - S[1]) / (E[1] - S[1]) * (E[0] - S[0]), Y)

    poly = clip(poly, lambda P: P[0] >= x0, ix(x0))
    poly = clip(poly, lambda P: P[0] <= x1, ix(x1))
    poly = clip(poly, lambda P: P[1] >= y0, iy(y0))
    poly = clip(poly, lambda P: P[1] <= y1, iy(y1))
    return poly


# ---------------------------------------------------------------- integration

def integrate_poly_triangle(p, A, B, C):
    """Exact integral of p(y1, y2) over triangle ABC."""
    X = padd({(0, 0): A[0]}, padd({(1, 0): B[0] - A[0]}, {(0, 1): C[0] - A[0]}))
    Y = padd({(0, 0): A[1]}, padd({(1, 0): B[1] - A[1]}, {(0, 1): C[1] - A[1]}))
    q = compose_affine(p, X, Y)
    det = abs((B[0] - A[0]) * (C[1] - A[1]) - (B[1] - A[1]) * (C[0] - A[0]))
    tot = Fr(0)
    for (a, b), c in q.items():
        tot += c * Fr(math.factorial(a) * math.factorial(b), math.factorial(a + b + 2))
    return det * tot


def exact_siac(V, T, fields, k, h, coeffs, x, periodic=3, L=(Fr(1), Fr(1)), coeffs_y=None):
    """u*(x) exactly.  V: list of (Fr, Fr); T: list of index triples; fields[t]: poly dict.
    coeffs_y: the y-axis kernel's coefficients if they differ from the x-axis' (one-sided
    kernels, written on the symmetric node grid at the effective point)."""
    h = Fr(h)
    x1, x2 = Fr(x[0]), Fr(x[1])
    kp = kernel_cell_polys(k, coeffs)
    kpy = kp if coeffs_y is None else kernel_cell_polys(k, coeffs_y)
    nc = 3 * k + 1
    tb = [Fr(-(3 * k + 1), 2) + i for i in range(nc + 1)]
    # K_i((y - x1)/h) as a polynomial in y1 (resp. y2)
    def kpoly_in(var, xc, i):
        lin = {(1, 0): 1 / h, (0, 0): -xc / h} if var == 0 else {(0, 1): 1 / h, (0, 0): -xc / h}
        out = {}
        for m, c in enumerate((kp if var == 0 else kpy)[i]):
            if c != 0:
                out = padd(out, {mm: c * v for mm, v in ppow(lin, m).items()})
        return out

    KX = [kpoly_in(0, x1, i) for i in range(nc)]
    KY = [kpoly_in(1, x2, j) for j in range(nc)]
    shifts = [(sx, sy) for sx in ((-1, 0, 1) if periodic & 1 else (0,))
              for sy in ((-1, 0, 1) if periodic & 2 else (0,))]
    total = Fr(0)
    for t, tri in enumerate(T):
        for (sx, sy) in shifts:
            ox, oy = sx * L[0], sy * L[1]
            P = [(V[v][0] + ox, V[v][1] + oy) for v in tri]
            # u_t(y - s) as a polynomial in y
            sh = compose_affine(fields[t], {(1, 0): Fr(1), (0, 0): -ox}, {(0, 1): Fr(1), (0, 0): -oy})
            sh = {m: c for m, c in sh.items() if c != 0}
            for i in range(nc):
                cx0, cx1 = x1 + h * tb[i], x1 + h * tb[i + 1]
                if max(p[0] for p in P) <= cx0 or min(p[0] for p in P) >= cx1:
                    continue
                for j in range(nc):
                    cy0, cy1 = x2 + h * tb[j], x2 + h * tb[j + 1]
                    if max(p[1] for p in P) <= cy0 or min(p[1] for p in P) >= cy1:
                        continue
                    poly = clip_rect(list(P), cx0, cx1, cy0, cy1)
                    if len(poly) < 3:
                        continue
                    integrand = pmul(pmul(KX[i], KY[j]), sh)
                    for m in range(1, len(poly) - 1):
                        total += integrate_poly_triangle(integrand, poly[0], poly[m], poly[m + 1])
    return total / (h * h)
