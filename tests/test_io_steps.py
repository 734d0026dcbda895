"""Steps either side of the SIAC path: L2 projection of
a field into the orthonormal Dubiner modes, element point mapping and error norms, all on the
GPU through the C ABI (csrc/siac_io.cu).  References: the seeded input generator's numpy
projection (inputs.project, the same definition written independently), exactness on
polynomials, closed-form moments of the unit triangle and numpy reductions."""
import math

import numpy as np
import pytest

from paper_conf_sc_0007k13_b200 import inputs, siac


@pytest.mark.parametrize("n", [1, 2, 5, 10])
def test_projection_rule_moments(n):
    """sum_q w_q r^a s^b = 4 a! b! / (a+b+2)! (reference triangle = 4 x unit triangle) for
    a + b <= 2n - 2; weights sum to the reference area 2 (host call, no device)."""
    siac.build()
    rs, w = siac.projection_rule(n)
    assert rs.shape == (n * n, 2) and np.all(rs >= 0) and np.all(rs.sum(1) <= 1 + 1e-15)
    assert abs(w.sum() - 2.0) < 1e-14
    for a in range(2 * n - 1):
        for b in range(2 * n - 1 - a):
            exact = 4.0 * math.factorial(a) * math.factorial(b) / math.factorial(a + b + 2)
            got = np.sum(w * rs[:, 0] ** a * rs[:, 1] ** b)
            assert abs(got - exact) <= 1e-14 * max(1.0, exact), (a, b)


def _gpu_project(w, k, n_quad, f_torch):
    import torch
    dev = torch.device("cuda", 0)
    rs, _ = siac.projection_rule(n_quad)
    d_V = torch.from_numpy(np.ascontiguousarray(w.V)).to(dev)
    d_T = torch.from_numpy(np.ascontiguousarray(w.T.astype(np.int32))).to(dev)
    d_rs = torch.from_numpy(rs).to(dev)
    d_P = torch.empty((len(w.T) * n_quad * n_quad, 2), dtype=torch.float64, device=dev)
    siac.map_points_async(d_V, d_T, d_rs, d_P)
    d_f = f_torch(d_P[:, 0], d_P[:, 1]).contiguous()
    d_c = torch.empty((len(w.T), inputs.n_modes(k)), dtype=torch.float64, device=dev)
    siac.project_async(k, n_quad, d_f, d_c)
    torch.cuda.synchronize()
    return d_P.cpu().numpy(), d_c.cpu().numpy()


@pytest.mark.gpu
@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_project_matches_numpy_projection(k):
    import torch
    w = inputs.make_config(2)
    P, c = _gpu_project(w, k, 10, lambda x, y: torch.sin(2 * math.pi * x) * torch.sin(2 * math.pi * y))
    ref = inputs.project(w.V, w.T, k, inputs.sinsin, n_quad=10)
    assert np.abs(c - ref).max() <= 1e-13 * np.abs(ref).max()
    # the mapped points are the rule nodes in every element
    rs, _ = siac.projection_rule(10)
    v0 = w.V[w.T[:, 0]]
    e1, e2 = w.V[w.T[:, 1]] - v0, w.V[w.T[:, 2]] - v0
    Pn = v0[:, None] + rs[None, :, 0:1] * e1[:, None] + rs[None, :, 1:2] * e2[:, None]
    assert np.abs(P - Pn.reshape(-1, 2)).max() < 1e-15


@pytest.mark.gpu
@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_project_reproduces_polynomials(k):
    """A global polynomial of degree <= k is in P_k on every element: its projection evaluated
    anywhere in an element equals it (exact up to rounding)."""
    import torch
    rng = np.random.default_rng(7 + k)
    terms = [(a, b, rng.uniform(-1, 1)) for a in range(k + 1) for b in range(k + 1 - a)]

    def f_np(x, y):
        return sum(c * x ** a * y ** b for a, b, c in terms)

    w = inputs.make_config(2)
    _, c = _gpu_project(w, k, k + 2, lambda x, y: sum(cc * x ** a * y ** b for a, b, cc in terms))
    xi, eta = rng.uniform(-1, 1, (2, 64))
    keep = xi + eta <= 0
    xi, eta = xi[keep], eta[keep]
    Phi = inputs.dubiner_eval(k, xi, eta)               # (m, nb)
    r, s = (xi + 1) / 2, (eta + 1) / 2
    for t in range(0, len(w.T), 97):
        v0, v1, v2 = w.V[w.T[t]]
        X = v0[0] + r * (v1[0] - v0[0]) + s * (v2[0] - v0[0])
        Y = v0[1] + r * (v1[1] - v0[1]) + s * (v2[1] - v0[1])
        assert np.abs(Phi @ c[t] - f_np(X, Y)).max() < 1e-12


@pytest.mark.gpu
def test_error_norms_match_numpy_and_are_deterministic():
    import torch
    rng = np.random.default_rng(3)
    n = 1_000_003
    u, ref, wt = rng.normal(size=n), rng.normal(size=n), rng.uniform(0, 1, n)
    d = [torch.from_numpy(a).cuda() for a in (u, ref, wt)]
    out = torch.empty(3, dtype=torch.float64, device="cuda")
    siac.error_norms_async(d[0], d[1], d[2], out)
    a = out.cpu().numpy().copy()
    siac.error_norms_async(d[0], d[1], d[2], out)
    b = out.cpu().numpy()
    assert np.array_equal(a, b)
    e = u - ref
    assert abs(a[0] - math.sqrt(np.sum(wt * e * e))) <= 1e-13 * a[0]
    assert a[1] == np.abs(e).max()
    assert abs(a[2] - wt.sum()) <= 1e-13 * a[2]
    siac.error_norms_async(d[0], d[1], None, out)
    c = out.cpu().numpy()
    assert abs(c[0] - math.sqrt(np.sum(e * e))) <= 1e-13 * c[0] and c[2] == n


@pytest.mark.gpu
def test_filtered_error_pipeline_on_gpu():
    """project -> siac_eval -> error norms, all on the device: the filtered L2 error of
    sin(2 pi x) sin(2 pi y) (cfg 1 mesh, k = 1) is below the projection error (the filter's
    purpose, L179-185) and matches the host-side computation."""
    import torch
    w = inputs.make_config(1)
    k = w.k
    _, c = _gpu_project(w, k, 10, lambda x, y: torch.sin(2 * math.pi * x) * torch.sin(2 * math.pi * y))
    ctx = siac.create(w.V, w.T, c, k, w.h, periodic=3, device=0)
    P = torch.from_numpy(w.points).cuda()
    u = torch.empty(w.n_points, dtype=torch.float64, device="cuda")
    ctx.eval_async(P, u)
    ex = torch.sin(2 * math.pi * P[:, 0]) * torch.sin(2 * math.pi * P[:, 1])
    out = torch.empty(3, dtype=torch.float64, device="cuda")
    siac.error_norms_async(u, ex, None, out)
    torch.cuda.synchronize()
    ctx.destroy()
    e = (u - ex).cpu().numpy()
    got = out.cpu().numpy()
    assert abs(got[1] - np.abs(e).max()) <= 1e-15
    # unfiltered dG error at the same points
    xi_eta = 2 * np.asarray(inputs.EVAL_RULES[k], dtype=np.float64) - 1
    Phi = inputs.dubiner_eval(k, xi_eta[:, 0], xi_eta[:, 1])
    udg = (c @ Phi.T).reshape(-1)
    e_dg = np.abs(udg - ex.cpu().numpy()).max()
    assert got[1] < 0.5 * e_dg
