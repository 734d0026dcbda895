"""CPU-side checks of the C ABI: the library builds for sm_100a, loads, exports every symbol
include/siac.h declares, and validates arguments before touching a device."""
import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_sc_0007k13_b200 import inputs, siac

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    siac.build()
    return siac.lib()


def _declared():
    txt = open(os.path.join(ROOT, "include", "siac.h")).read()
    return sorted(set(re.findall(r"^\s*(?:siac_status|void|const char \*)\s*(siac3?_\w+)\s*\(", txt, re.M)))


def test_header_declares_expected_calls():
    names = _declared()
    assert set(names) == set(siac.EXPORTED), names


def test_library_exports_every_declared_symbol(L):
    for name in _declared():
        assert hasattr(L, name), name
    assert "sm_100a" in siac.version()


def test_library_contains_sm100a_code(L):
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", siac.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def _params(**kw):
    p = dict(k=1, h=0.05, periodic=3, domain=(0.0, 0.0, 1.0, 1.0), device=0, cell_factor=0.0)
    p.update(kw)
    return p


@pytest.mark.parametrize("bad,msg", [
    (dict(k=0), "k must"), (dict(k=5), "k must"), (dict(h=-1.0), "h must"), (dict(h=float("nan")), "h must"),
    (dict(h=0.3), "exceeds the periodic"), (dict(domain=(0.0, 0.0, -1.0, 1.0)), "domain"),
    (dict(periodic=4), "periodic"), (dict(basis=2), "basis"), (dict(boundary=2), "boundary"),
])
def test_create_rejects_bad_params(L, bad, msg):
    V, T = inputs.structured_mesh(4)
    C = np.zeros((len(T), 3))
    with pytest.raises(siac.SiacError, match=msg):
        siac.create(V, T, C, **_params(**bad))


def test_create_rejects_bad_mesh(L):
    V, T = inputs.structured_mesh(4)
    C = np.zeros((len(T), 3))
    T2 = T.copy()
    T2[3, 1] = 999
    with pytest.raises(siac.SiacError, match="index out of range"):
        siac.create(V, T2, C, **_params())
    T3 = T.copy()
    T3[0] = [0, 1, 2]              # collinear bottom-row vertices
    with pytest.raises(siac.SiacError, match="zero-area"):
        siac.create(V, T3, C, **_params())
    V2 = V.copy()
    V2[5, 0] = 1.5
    with pytest.raises(siac.SiacError, match="outside the periodic"):
        siac.create(V2, T, C, **_params())
    C2 = C.copy()
    C2[2, 1] = np.inf
    with pytest.raises(siac.SiacError, match="non-finite coefficient"):
        siac.create(V, T, C2, **_params())


def test_null_context_is_einval(L):
    assert L.siac_eval(None, None, 0, None) == -1
    assert L.siac_destroy(None) is None


def test_create_without_gpu_reports_device_error(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    V, T = inputs.structured_mesh(4)
    with pytest.raises(siac.SiacError, match="siac error -4"):
        siac.create(V, T, np.zeros((len(T), 3)), **_params())


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_host_kernel_cell_table(L, oracle_mod, k):
    """The library's exact per-cell kernel polynomials equal K evaluated by the oracle."""
    tbl, _ = siac.host_tables(k)
    tau = np.linspace(-0.499, 0.499, 37)
    for i in range(3 * k + 1):
        t = -(3 * k + 1) / 2 + i + 0.5 + tau
        poly = sum(tbl[i, m] * tau ** m for m in range(k + 1))
        assert np.abs(poly - oracle_mod.kernel_values(k, t)).max() < 1e-14


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_host_basis_matrix(L, k):
    """Row i of the Dubiner->centred-monomial matrix reproduces mode i (scipy evaluation)."""
    _, R = siac.host_tables(k)
    order = [(a, b) for a in range(k, -1, -1) for b in range(k - a + 1)]
    rng = np.random.default_rng(0)
    r, s = rng.uniform(0, 0.5, (2, 50))
    rho, sig = 3 * r - 1, 3 * s - 1
    mono = np.stack([rho ** a * sig ** b for a, b in order], axis=1)
    ref = inputs.dubiner_eval(k, 2 * r - 1, 2 * s - 1)
    assert np.abs(mono @ R.T - ref).max() < 1e-12


def test_tet_rule_exact(L):
    """siac3_tet_rule (host): the collapsed Gauss-Jacobi rule on the unit tetrahedron integrates
    r^a s^b t^c exactly up to degree 2n-1: a! b! c! / (a+b+c+3)! (Dirichlet integral)."""
    from math import factorial
    for n in (2, 4, 5):
        q = siac.tet_rule(n)
        assert q.shape == (n ** 3, 4) and np.all(q[:, 3] > 0)
        for a in range(2 * n):
            for b in range(2 * n - a):
                for c in range(2 * n - a - b):
                    exact = factorial(a) * factorial(b) * factorial(c) / factorial(a + b + c + 3)
                    got = np.sum(q[:, 3] * q[:, 0] ** a * q[:, 1] ** b * q[:, 2] ** c)
                    assert abs(got - exact) < 1e-15 + 1e-13 * exact, (n, a, b, c)
