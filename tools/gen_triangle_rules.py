#!/usr/bin/env python3
"""Generate fully symmetric quadrature rules on the triangle (Dunavant-type orbit structures).

Used for two unrelated purposes:
  * the GPU path's sub-triangle quadrature (exact for total degree 3k, the degree of the
    integrand K_x * K_y * u on a sub-triangle: PAPER.md §2.2, Eq. (2)),
    written to paper_conf_sc_0007k13_b200/csrc/siac_quadrature.h;
  * the evaluation-point layouts (degree-2k rules, "the quadrature points of the polynomial
    interpolant defined over each element"), written to
    paper_conf_sc_0007k13_b200/inputs/eval_rules.py.

The oracle does NOT use any of these tables (it integrates trapezoids with tensor
Gauss-Legendre rules), so the two sides stay independent.

Each rule is found by Newton/Gauss-Newton on the moment equations
    sum_i w_i r_i^p s_i^q = 2 p! q! / (p+q+2)!     (weights normalised to sum 1)
for all p+q <= degree, in 60-digit mpmath arithmetic, starting from the classical
orbit structure and approximate node positions (Dunavant 1985 orbit counts).
The script then re-verifies exactness in exact rational arithmetic against the
rounded float64 values (residual must be <= 1e-15) before writing anything.

Usage: python tools/gen_triangle_rules.py
"""
import math
import os
import sys
from fractions import Fraction

import mpmath as mp

mp.mp.dps = 60

# orbit specs: ("S3", w) | ("S21", a, w) | ("S111", a, b, w); a,b barycentric coords
START = {
    2: [("S21", 1 / 6, 1 / 3)],
    3: [("S3", -27 / 48), ("S21", 0.2, 25 / 48)],
    4: [("S21", 0.445948490915965, 0.223381589678011),
        ("S21", 0.091576213509771, 0.109951743655322)],
    6: [("S21", 0.249286745170910, 0.116786275726379),
        ("S21", 0.063089014491502, 0.050844906370207),
        ("S111", 0.053145049844817, 0.310352451033784, 0.082851075618374)],
    8: [("S3", 0.144315607677787),
        ("S21", 0.459292588292723, 0.095091634267285),
        ("S21", 0.170569307751760, 0.103217370534718),
        ("S21", 0.050547228317031, 0.032458497623198),
        ("S111", 0.008394777409958, 0.263112829634638, 0.027230314174435)],
    9: [("S3", 0.097135796282799),
        ("S21", 0.489682519198738, 0.031334700227139),
        ("S21", 0.437089591492937, 0.077827541004774),
        ("S21", 0.188203535619033, 0.079647738927210),
        ("S21", 0.044729513394453, 0.025577675658698),
        ("S111", 0.036838412054736, 0.221962989160766, 0.043283539377289)],
    12: [("S21", 0.488217389773805, 0.025731066440455),
         ("S21", 0.439724392294460, 0.043692544538038),
         ("S21", 0.271210385012116, 0.062858224217885),
         ("S21", 0.127576145541586, 0.034796112930709),
         ("S21", 0.021317350453210, 0.006166261051559),
         ("S111", 0.115343494534698, 0.275713269685514, 0.040371557766381),
         ("S111", 0.022838332222257, 0.281325580989940, 0.022356773202303),
         ("S111", 0.025734050548330, 0.116251915907597, 0.017316231108659)],
}


def unpack(spec):
    params, kinds = [], []
    for o in spec:
        kinds.append(o[0])
        params.extend(mp.mpf(v) for v in o[1:])
    return kinds, params


def expand(kinds, params):
    """-> list of (r, s, w) with (r, s) = barycentric coords 2 and 3 (unit triangle)."""
    pts, i = [], 0
    for kd in kinds:
        if kd == "S3":
            w = params[i]; i += 1
            t = mp.mpf(1) / 3
            pts.append((t, t, w))
        elif kd == "S21":
            a, w = params[i], params[i + 1]; i += 2
            c = 1 - 2 * a
            for bary in ((a, a, c), (a, c, a), (c, a, a)):
                pts.append((bary[1], bary[2], w))
        else:
            a, b, w = params[i], params[i + 1], params[i + 2]; i += 3
            c = 1 - a - b
            for bary in ((a, b, c), (a, c, b), (b, a, c), (b, c, a), (c, a, b), (c, b, a)):
                pts.append((bary[1], bary[2], w))
    return pts


def exact_moment(p, q):
    return Fraction(2 * math.factorial(p) * math.factorial(q), math.factorial(p + q + 2))


def residual(kinds, params, deg):
    pts = expand(kinds, params)
    res = []
    for p in range(deg + 1):
        for q in range(deg + 1 - p):
            s = mp.fsum(w * r ** p * t ** q for (r, t, w) in pts)
            e = exact_moment(p, q)
            res.append(s - mp.mpf(e.numerator) / e.denominator)
    return res


def solve(deg):
    kinds, params = unpack(START[deg])
    n = len(params)
    for it in range(60):
        F = residual(kinds, params, deg)
        nrm = max(abs(f) for f in F)
        if nrm < mp.mpf(10) ** -50:
            break
        h = mp.mpf(10) ** -30
        J = []
        for j in range(n):
            pp = list(params); pp[j] += h
            Fp = residual(kinds, pp, deg)
            J.append([(Fp[i] - F[i]) / h for i in range(len(F))])
        # Gauss-Newton: (J^T J) d = -J^T F
        JT = mp.matrix(J)             # n x m
        A = JT * JT.T
        b = JT * mp.matrix(F)
        d = mp.lu_solve(A, -b)
        params = [params[j] + d[j] for j in range(n)]
    F = residual(kinds, params, deg)
    nrm = max(abs(f) for f in F)
    if nrm > mp.mpf(10) ** -40:
        raise SystemExit(f"degree {deg}: Newton did not converge (residual {nrm})")
    pts = expand(kinds, params)
    for (r, s, w) in pts:
        if not (r > 0 and s > 0 and r + s < 1):
            raise SystemExit(f"degree {deg}: node outside the triangle")
    return pts


def verify_float(pts, deg):
    worst = 0.0
    for p in range(deg + 1):
        for q in range(deg + 1 - p):
            s = sum(Fraction(float(w)) * Fraction(float(r)) ** p * Fraction(float(t)) ** q
                    for (r, t, w) in pts)
            e = exact_moment(p, q)
            worst = max(worst, abs(float((s - e) / e)))
    if worst > 1e-14:
        raise SystemExit(f"degree {deg}: float64 rounding residual {worst}")
    return worst


def fmt(x):
    return repr(float(x))


def main():
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    rules = {}
    for deg in sorted(START):
        pts = solve(deg)
        worst = verify_float(pts, deg)
        rules[deg] = pts
        print(f"degree {deg:2d}: {len(pts):2d} points, float64 moment residual {worst:.2e}", file=sys.stderr)

    # --- GPU sub-triangle quadrature (degree 3k) ---
    hdr = os.path.join(root, "paper_conf_sc_0007k13_b200", "csrc", "siac_quadrature.h")
    with open(hdr, "w") as f:
        f.write("// GENERATED by tools/gen_triangle_rules.py -- do not edit.\n")
        f.write("// Fully symmetric triangle rules exact for total degree 3k (k = 1..4), the degree of\n")
        f.write("// K_x(z1) K_y(z2) u(z) on one fan sub-triangle (PAPER.md L236-280, Eq. (2); SURVEY Q11).\n")
        f.write("// Nodes are (r, s) on the unit triangle {r,s >= 0, r+s <= 1}; weights sum to 1, so\n")
        f.write("// integral over a sub-triangle = area * sum_q w_q f(P0 + r_q E1 + s_q E2).\n")
        f.write("#pragma once\n\n")
        for k in (1, 2, 3, 4):
            pts = rules[3 * k]
            f.write(f"#define SIAC_NQ_K{k} {len(pts)}\n")
            f.write(f"__constant__ double siac_qr_k{k}[{len(pts)}] = {{{', '.join(fmt(p[0]) for p in pts)}}};\n")
            f.write(f"__constant__ double siac_qs_k{k}[{len(pts)}] = {{{', '.join(fmt(p[1]) for p in pts)}}};\n")
            f.write(f"__constant__ double siac_qw_k{k}[{len(pts)}] = {{{', '.join(fmt(p[2]) for p in pts)}}};\n\n")
    # --- evaluation point layouts (degree 2k) ---
    py = os.path.join(root, "paper_conf_sc_0007k13_b200", "inputs", "eval_rules.py")
    with open(py, "w") as f:
        f.write('"""GENERATED by tools/gen_triangle_rules.py -- do not edit.\n\n')
        f.write("Evaluation-point layouts: nodes of the fully symmetric degree-2k triangle rule\n")
        f.write("(3/6/12/16 points for k=1..4). PAPER.md L313-314: the computation grid is the\n")
        f.write("element quadrature points; the rule is unspecified, SURVEY Q7 fixes degree 2k.\n")
        f.write('Nodes are (r, s) on the unit triangle; weights are included for completeness."""\n\n')
        f.write("EVAL_RULES = {\n")
        for k in (1, 2, 3, 4):
            pts = rules[2 * k]
            f.write(f"    {k}: [\n")
            for (r, s, w) in pts:
                f.write(f"        ({fmt(r)}, {fmt(s)}, {fmt(w)}),\n")
            f.write("    ],\n")
        f.write("}\n")
    print("wrote", hdr, "and", py, file=sys.stderr)


if __name__ == "__main__":
    main()
