"""Input generators (meshes, points, projection) and the generated triangle rules."""
import math
import os
import re
from fractions import Fraction

import numpy as np
import pytest

from paper_conf_sc_0007k13_b200 import inputs
from paper_conf_sc_0007k13_b200.inputs.eval_rules import EVAL_RULES

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _exact_moment(p, q):
    return Fraction(2 * math.factorial(p) * math.factorial(q), math.factorial(p + q + 2))


def _check_rule(r, s, w, deg):
    worst = 0.0
    for p in range(deg + 1):
        for q in range(deg + 1 - p):
            tot = sum(Fraction(wi) * Fraction(ri) ** p * Fraction(si) ** q for ri, si, wi in zip(r, s, w))
            worst = max(worst, abs(float(tot / _exact_moment(p, q) - 1)))
    return worst


def _parse_header():
    txt = open(os.path.join(ROOT, "paper_conf_sc_0007k13_b200", "csrc", "siac_quadrature.h")).read()
    rules = {}
    for k in (1, 2, 3, 4):
        arr = {}
        for nm in ("qr", "qs", "qw"):
            m = re.search(rf"siac_{nm}_k{k}\[\d+\] = \{{([^}}]*)\}}", txt)
            arr[nm] = [float(x) for x in m.group(1).split(",")]
        rules[k] = arr
    return rules


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_gpu_subtriangle_rule_exact_degree_3k(k):
    """The GPU quadrature must integrate K_x K_y u (total degree 3k) exactly."""
    R = _parse_header()[k]
    assert len(R["qr"]) == {1: 4, 2: 12, 3: 19, 4: 33}[k]
    assert _check_rule(R["qr"], R["qs"], R["qw"], 3 * k) < 1e-14
    # and not exact one degree higher for k >= 2 (the rule is not over-sized by accident)
    if k >= 2:
        assert _check_rule(R["qr"], R["qs"], R["qw"], 3 * k + 1) > 1e-8


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_eval_rules(k):
    rule = EVAL_RULES[k]
    assert len(rule) == {1: 3, 2: 6, 3: 12, 4: 16}[k]
    r, s, w = zip(*rule)
    assert _check_rule(r, s, w, 2 * k) < 1e-14
    assert all(ri > 0 and si > 0 and ri + si < 1 for ri, si in zip(r, s))


def test_structured_mesh():
    V, T = inputs.structured_mesh(20)
    assert len(T) == 800
    A = inputs.triangle_areas(V, T)
    assert np.allclose(A, 1 / 800, rtol=1e-12)
    assert inputs.max_edge(V, T) == pytest.approx(math.sqrt(2) / 20)


@pytest.mark.parametrize("graded", [False, True])
def test_delaunay_mesh_covers_unit_square(graded):
    V, T = inputs.lattice_delaunay_mesh(4096, seed=3, graded=graded)
    A = inputs.triangle_areas(V, T)
    assert abs(A.sum() - 1.0) < 1e-12
    assert 3500 < len(T) < 4700
    assert V.min() >= 0.0 and V.max() <= 1.0
    # periodic-compatible: boundary nodes on opposite sides coincide
    for ax in (0, 1):
        lo = np.sort(V[V[:, ax] == 0.0][:, 1 - ax])
        hi = np.sort(V[V[:, ax] == 1.0][:, 1 - ax])
        assert np.array_equal(lo, hi)
    # determinism
    V2, T2 = inputs.lattice_delaunay_mesh(4096, seed=3, graded=graded)
    assert np.array_equal(V, V2) and np.array_equal(T, T2)


def test_graded_mesh_size_variation():
    V, T = inputs.lattice_delaunay_mesh(16384, seed=1003, graded=True)
    e = np.linalg.norm(V[T[:, 1]] - V[T[:, 0]], axis=1)
    assert e.max() / np.median(e) > 2.5


def test_eval_points_inside_elements():
    V, T = inputs.lattice_delaunay_mesh(1000, seed=1)
    for k in (1, 2, 3, 4):
        P = inputs.eval_points(V, T, k).reshape(len(T), -1, 2)
        v0, v1, v2 = V[T[:, 0]], V[T[:, 1]], V[T[:, 2]]
        for j in range(P.shape[1]):
            d = P[:, j] - v0
            a, b = v1 - v0, v2 - v0
            det = a[:, 0] * b[:, 1] - a[:, 1] * b[:, 0]
            r = (b[:, 1] * d[:, 0] - b[:, 0] * d[:, 1]) / det
            s = (-a[:, 1] * d[:, 0] + a[:, 0] * d[:, 1]) / det
            assert np.all(r > 0) and np.all(s > 0) and np.all(r + s < 1)


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_projection_reproduces_polynomials(k):
    """L2 projection onto P_k is the identity on P_k."""
    V, T = inputs.lattice_delaunay_mesh(200, seed=2)
    f = lambda x, y: (0.3 + x - 2 * y) ** k + 0.5 * x * y ** (k - 1)  # noqa: E731
    C = inputs.project(V, T, k, f)
    xi, eta = np.array([-0.5, -0.2, 0.1]), np.array([-0.4, 0.0, -0.7])
    Phi = inputs.dubiner_eval(k, xi, eta)
    r, s = (xi + 1) / 2, (eta + 1) / 2
    v0, v1, v2 = V[T[:, 0]], V[T[:, 1]], V[T[:, 2]]
    X = v0[:, None, 0] + r * (v1 - v0)[:, None, 0] + s * (v2 - v0)[:, None, 0]
    Y = v0[:, None, 1] + r * (v1 - v0)[:, None, 1] + s * (v2 - v0)[:, None, 1]
    assert np.abs(C @ Phi.T - f(X, Y)).max() < 1e-12


def test_configs_small():
    w = inputs.make_config(1)
    assert len(w.T) == 800 and w.n_points == 2400 and w.h == 0.05
    w2 = inputs.make_config(2)
    assert w2.k == 2 and w2.n_points == 6 * len(w2.T)
    assert (3 * w2.k + 1) * w2.h < 1.0
