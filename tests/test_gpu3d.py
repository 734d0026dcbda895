"""GPU parity of the tetrahedral path (siac3_*) against
the 3D oracle, element by element, through the C ABI.  Tolerance: north_star's rule (1e-10
normwise and pointwise where |o| >= 1e-2 max|o|)."""
import numpy as np
import pytest

from paper_conf_sc_0007k13_b200.inputs import mesh3d as m3

from test_gpu_parity import assert_parity

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def siac_mod():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_sc_0007k13_b200 import siac
    siac.lib()
    return siac


def _h(V, T, k):
    """h = the largest tetrahedron extent (the 2D configs' h = max edge), capped so that the
    stencil W = (3k+1)h fits the unit period."""
    return min(m3.max_extent3(V, T), 0.95 / (3 * k + 1))


def _eval(siac_mod, V, T, C, k, h, P, periodic=7):
    ctx = siac_mod.create3(V, T, C, k, h, periodic=periodic)
    try:
        return ctx.eval(P)
    finally:
        ctx.destroy()


@pytest.mark.parametrize("k", [1, 2, 3])
def test_constant_field_every_point(siac_mod, k):
    """u = 1 -> u* = 1 at every element point (periodic Delaunay mesh): the splitting of every
    tetrahedron into kernel-cell pieces covers the stencil exactly."""
    V, T = m3.lattice_delaunay_mesh3({1: 3000, 2: 8000, 3: 12000}[k], seed=10 + k)
    C = np.zeros((len(T), m3.n_modes3(k)))
    C[:, 0] = 1.0
    h = _h(V, T, k)
    P = m3.eval_points3(V, T)[:: {1: 1, 2: 2, 3: 40}[k]]
    g = _eval(siac_mod, V, T, C, k, h, P)
    assert np.abs(g - 1).max() < 1e-12


@pytest.mark.parametrize("k,mesh,periodic", [(1, "d", 7), (2, "d", 7), (3, "s", 7), (1, "d", 0), (2, "s", 5)])
def test_parity_random_field(siac_mod, oracle_mod, k, mesh, periodic):
    if mesh == "d":
        V, T = m3.lattice_delaunay_mesh3(2000 if k == 1 else 4000, seed=20 + k)
        h = _h(V, T, k)
    else:
        V, T = m3.structured_mesh3(3 if k == 3 else 5)
        h = 0.1 if k == 3 else 0.13
    C = m3.random_modes3(len(T), k, seed=30 + k)
    P = m3.eval_points3(V, T)[:: max(1, len(T) // (6 if k == 1 else 3))]
    P = np.concatenate([P, [[0, 0, 0], [1, 1, 1], [0.5, 0, 1]]])
    g = _eval(siac_mod, V, T, C, k, h, P, periodic)
    o = oracle_mod.oracle_eval3(V, T, C, k, h, P, periodic=periodic)
    assert_parity(g, o)


def test_small_h_deep_splits(siac_mod, oracle_mod):
    """h smaller than the tetrahedra: several planes per axis cut each tetrahedron."""
    V, T = m3.structured_mesh3(3)
    C = m3.random_modes3(len(T), 1, seed=3)
    h = 0.45 / 3
    P = np.random.default_rng(4).uniform(0, 1, (12, 3))
    g = _eval(siac_mod, V, T, C, 1, h, P)
    assert_parity(g, oracle_mod.oracle_eval3(V, T, C, 1, h, P))


def test_polynomial_reproduction_and_superconvergence(siac_mod):
    """A global P1 field is reproduced at interior points (non-periodic), and the filtered error
    on sin sin sin decays at order >= 2k+1 - 0.2 on structured meshes (k = 1)."""
    V, T = m3.lattice_delaunay_mesh3(6000, seed=5)
    f = lambda x, y, z: 0.3 + x - 0.2 * y + 0.7 * z  # noqa: E731
    C = m3.project3(V, T, 1, f)
    h = 0.05
    P = np.random.default_rng(6).uniform(0.15, 0.85, (200, 3))
    g = _eval(siac_mod, V, T, C, 1, h, P, periodic=0)
    assert np.abs(g - f(P[:, 0], P[:, 1], P[:, 2])).max() < 1e-12
    errs = []
    for N in (8, 16, 32):
        V, T = m3.structured_mesh3(N)
        C = m3.project3(V, T, 1, m3.sin3)
        P = m3.eval_points3(V, T)[:: 37]
        g = _eval(siac_mod, V, T, C, 1, 1.0 / N, P)
        errs.append(np.abs(g - m3.sin3(P[:, 0], P[:, 1], P[:, 2])).max())
    rates = [np.log2(errs[i] / errs[i + 1]) for i in range(2)]
    assert min(rates) >= 2.8, (errs, rates)


def test_async_and_counters(siac_mod):
    import torch
    V, T = m3.lattice_delaunay_mesh3(1500, seed=8)
    C = m3.random_modes3(len(T), 2, seed=9)
    h = _h(V, T, 2)
    P = m3.eval_points3(V, T)
    ctx = siac_mod.create3(V, T, C, 2, h)
    ref = ctx.eval(P)
    ctx.set_counting(True)
    d = torch.from_numpy(P).cuda()
    o = torch.empty(len(P), dtype=torch.float64, device="cuda")
    s = torch.cuda.Stream()
    ctx.eval_async(d, o, s)
    s.synchronize()
    st = ctx.stats()
    ctx.destroy()
    assert np.array_equal(o.cpu().numpy(), ref)
    assert st["pieces"] >= st["pairs"] > 0


@pytest.mark.parametrize("k", [1, 2, 3])
def test_schedules_agree(siac_mod, oracle_mod, k):
    """Warp-per-tile (schedule 0, default) and thread-per-point (schedule 1) mappings of the same
    decomposition: equal to rounding, equal pair and piece counts, both at oracle parity
    (ragged last tile: the point count is not a multiple of 32).  k = 3 on the structured mesh with
    h = the tetrahedron extent (W = 10h covers most of the period: a few points only)."""
    if k < 3:
        V, T = m3.lattice_delaunay_mesh3({1: 1500, 2: 1200}[k], seed=40 + k)
        h = _h(V, T, k)
        P = m3.eval_points3(V, T)[:: {1: 5, 2: 11}[k]][:-3]
    else:
        V, T = m3.structured_mesh3(11)
        h = 1.0 / 11
        P = m3.eval_points3(V, T)[np.random.default_rng(43).choice(4 * len(T), 9, replace=False)]
    C = m3.random_modes3(len(T), k, seed=50 + k)
    vals, stats = [], []
    for sch in (0, 1):
        ctx = siac_mod.create3(V, T, C, k, h)
        ctx.set_schedule(sch)
        ctx.set_counting(True)
        vals.append(ctx.eval(P))
        stats.append(ctx.stats())
        ctx.destroy()
    assert stats[0] == stats[1], stats
    sc = np.abs(vals[1]).max()
    assert np.abs(vals[0] - vals[1]).max() <= 1e-13 * sc
    o = oracle_mod.oracle_eval3(V, T, C, k, h, P[:: max(1, len(P) // 16)])
    assert_parity(vals[0][:: max(1, len(P) // 16)], o)


def test_schedule_rejects_unknown(siac_mod):
    V, T = m3.structured_mesh3(2)
    C = m3.random_modes3(len(T), 1, seed=1)
    ctx = siac_mod.create3(V, T, C, 1, 0.2)
    with pytest.raises(Exception):
        ctx.set_schedule(2)
    ctx.destroy()


def test_points_outside_nonperiodic_domain(siac_mod, oracle_mod):
    """Zero extension on non-periodic axes: whole point tiles far outside the domain (empty
    candidate-cell ranges after clamping) give exactly 0; mixed tiles match the oracle."""
    V, T = m3.structured_mesh3(4)
    C = m3.random_modes3(len(T), 1, seed=61)
    rng = np.random.default_rng(62)
    far = rng.uniform(-9, -3, (40, 3))
    near = rng.uniform(-0.3, 1.3, (30, 3))
    P = np.concatenate([far, near])
    for sch in (0, 1):
        ctx = siac_mod.create3(V, T, C, 1, 0.2, periodic=0)
        ctx.set_schedule(sch)
        g = ctx.eval(P)
        ctx.destroy()
        assert np.all(g[:40] == 0.0)
        assert_parity(g[40:], oracle_mod.oracle_eval3(V, T, C, 1, 0.2, near, periodic=0))
