"""Pins for the oracle's kernel: B-spline values, coefficients, moments, Fourier symbol.

PAPER.md L196-208 (kernel definition), L250-254 (support (3k+1)h); SURVEY §8(c.4) P1, P2, P6.
"""
import math
import os
from fractions import Fraction

import numpy as np
import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _read(name):
    rows = []
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if line and not line.startswith("#"):
            rows.append(line.split())
    return rows


def test_bspline_textbook_values(oracle_mod):
    for k, t, v in _read("bspline_values.txt"):
        got = oracle_mod.bspline_values(int(k), np.array([float(Fraction(t))]))[0]
        assert got == pytest.approx(float(Fraction(v)), abs=1e-15), (k, t)


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_bspline_partition_of_unity_and_support(oracle_mod, k):
    t = np.linspace(-3.0, 3.0, 1001)
    s = sum(oracle_mod.bspline_values(k, t - j) for j in range(-8, 9))
    assert np.abs(s - 1.0).max() < 1e-14
    out = np.array([-(k + 1) / 2 - 0.3, (k + 1) / 2 + 0.01, 5.0])
    assert np.all(oracle_mod.bspline_values(k, out) == 0.0)


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_kernel_coefficients_match_literature(oracle_mod, k):
    gold = {int(r[0]): [Fraction(x) for x in r[1:]] for r in _read("kernel_coefficients.txt")}
    assert oracle_mod.kernel_coefficients(k) == gold[k]
    assert sum(gold[k]) == 1


def _kernel_moment_numeric(oracle_mod, k, m):
    """int K(t) t^m dt with the C kernel: Gauss-Legendre on every unit knot interval
    (K is a polynomial of degree k there, so 12 points are exact for m <= 2k+2+...)."""
    g, w = np.polynomial.legendre.leggauss(16)
    lo = -(3 * k + 1) / 2
    tot = 0.0
    for i in range(3 * k + 1):
        a = lo + i
        t = a + 0.5 * (1 + g)
        tot += 0.5 * np.sum(w * oracle_mod.kernel_values(k, t) * t ** m)
    return tot


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_kernel_moments(oracle_mod, k):
    """K reproduces polynomials of degree <= r = 2k by convolution:
    m_0 = 1, m_1..m_2k = 0 (m_{2k+1} = 0 by symmetry), and m_{2k+2} != 0."""
    assert _kernel_moment_numeric(oracle_mod, k, 0) == pytest.approx(1.0, abs=1e-14)
    for m in range(1, 2 * k + 2):
        assert abs(_kernel_moment_numeric(oracle_mod, k, m)) < 1e-12 * (3 * k) ** m
    mexact = {1: Fraction(-4, 15), 2: Fraction(3229, 1344), 3: Fraction(-1916, 45)}
    num = _kernel_moment_numeric(oracle_mod, k, 2 * k + 2)
    if k in mexact:
        assert num == pytest.approx(float(mexact[k]), rel=1e-11)
    else:
        assert num == pytest.approx(1249.167, rel=1e-6)


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_kernel_support(oracle_mod, k):
    """Supp K = (3k+1) in units of h."""
    half = (3 * k + 1) / 2
    assert np.all(oracle_mod.kernel_values(k, np.array([-half - 1e-9, half, half + 0.5, -50.0])) == 0.0)
    assert oracle_mod.kernel_values(k, np.array([half - 0.01]))[0] != 0.0


A2 = {  # K^(2 pi h), 20 digits
    1: {10: 0.99832821233897837058, 20: 0.99989271705617664757, 40: 0.99999325036512901561},
    2: {10: 0.99980943475118350282, 20: 0.99999685125577656528, 40: 0.99999995010802527194},
    3: {10: 0.99997719847663183783, 20: 0.99999990270935246393, 40: 0.99999999961147091008},
}


@pytest.mark.parametrize("k", [1, 2, 3])
def test_kernel_fourier_symbol(oracle_mod, k):
    """P6: int K(t) cos(w t) dt = sum_g c_g cos(w x_g) (sin(w/2)/(w/2))^(k+1) (the B-spline
    is the (k+1)-fold box convolution); checked against SURVEY A2's 20-digit values."""
    g, wq = np.polynomial.legendre.leggauss(40)
    c = [float(v) for v in oracle_mod.kernel_coefficients(k)]
    for N, expect in A2[k].items():
        w = 2 * math.pi / N
        lo = -(3 * k + 1) / 2
        num = 0.0
        for i in range(3 * k + 1):
            t = lo + i + 0.5 * (1 + g)
            num += 0.5 * np.sum(wq * oracle_mod.kernel_values(k, t) * np.cos(w * t))
        closed = sum(cg * math.cos(w * (gi - k)) for gi, cg in enumerate(c)) * (math.sin(w / 2) / (w / 2)) ** (k + 1)
        assert num == pytest.approx(expect, abs=2e-15)
        assert closed == pytest.approx(expect, abs=2e-15)
