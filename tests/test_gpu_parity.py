"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by element.

Tolerance (north_star: 1e-10 relative; rule from SURVEY §8(c.5)): PASS iff
    max_i |g_i - o_i| <= 1e-10 * max_i |o_i|                      (normwise), and
    |g_i - o_i| <= 1e-10 * |o_i|  for every i with |o_i| >= 1e-2 max|o|   (pointwise).
Small configs are compared at every point; the large ones evaluate ALL points on the GPU
in the bench's launch configuration and compare a deterministic sample the oracle can
afford, plus points next to the domain boundary (periodic wrap) and mesh vertices.
"""
import math

import numpy as np
import pytest

from paper_conf_sc_0007k13_b200 import inputs

pytestmark = pytest.mark.gpu

TOL = 1e-10


def assert_parity(g, o, tol=TOL):
    g, o = np.asarray(g), np.asarray(o)
    assert g.shape == o.shape
    assert np.all(np.isfinite(g))
    scale = max(np.abs(o).max(), 1e-300)
    err = np.abs(g - o)
    assert err.max() <= tol * scale, f"normwise {err.max() / scale:.3e}"
    big = np.abs(o) >= 1e-2 * scale
    if big.any():
        rel = err[big] / np.abs(o[big])
        assert rel.max() <= tol, f"pointwise {rel.max():.3e}"


@pytest.fixture(scope="module")
def siac_mod():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_sc_0007k13_b200 import siac
    siac.lib()
    return siac


_CFG = {}


def cfg(c, field="sinsin"):
    key = (c, field)
    if key not in _CFG:
        _CFG[key] = inputs.make_config(c, field_kind=field)
    return _CFG[key]


def gpu_eval(siac_mod, w, points=None, schedule=0, **kw):
    ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h, periodic=w.periodic, domain=w.domain, **kw)
    ctx.set_schedule(schedule)
    try:
        return ctx.eval(w.points if points is None else points)
    finally:
        ctx.destroy()


def sample_idx(n, m, seed):
    rng = np.random.default_rng(seed)
    return np.sort(rng.choice(n, size=min(n, m), replace=False))


# ------------------------------------------------------------------ configs

@pytest.mark.parametrize("field", ["sinsin", "random"])
def test_cfg1_every_point(siac_mod, oracle_mod, field):
    w = cfg(1, field)
    assert_parity(gpu_eval(siac_mod, w), oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points))


@pytest.mark.parametrize("field", ["sinsin", "random"])
def test_cfg2_every_point(siac_mod, oracle_mod, field):
    w = cfg(2, field)
    assert_parity(gpu_eval(siac_mod, w), oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points))


@pytest.mark.parametrize("c", [1, 2])
@pytest.mark.parametrize("schedule", [1, 2, 3, 4, 5, 6])
def test_every_schedule_matches_oracle(siac_mod, oracle_mod, c, schedule):
    """Every schedule (point, tile, warp-specialized, jump) computes the same values."""
    w = cfg(c, "random")
    o = oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points)
    assert_parity(gpu_eval(siac_mod, w, schedule=schedule), o)


@pytest.mark.parametrize("k", [1, 2, 3, 4])
@pytest.mark.parametrize("schedule", [2, 4, 5, 6])
def test_every_k_delaunay_random_field(siac_mod, oracle_mod, k, schedule):
    """Every degree on an unstructured periodic mesh, random modes, h = max edge: the jump
    schedule's corner polynomials and cross terms at every k against the oracle."""
    V, T = inputs.lattice_delaunay_mesh(1500, seed=20 + k)
    C = inputs.random_modes(len(T), k, seed=30 + k)
    h = inputs.max_edge(V, T)
    P = inputs.eval_points(V, T, k)[::5]
    ctx = siac_mod.create(V, T, C, k, h)
    ctx.set_schedule(schedule)
    g = ctx.eval(P)
    ctx.destroy()
    assert_parity(g, oracle_mod.oracle_eval(V, T, C, k, h, P))


@pytest.mark.parametrize("sch", [4, 5, 6])
@pytest.mark.parametrize("c,m", [(3, 400), (4, 150)])
def test_jump_and_tile_agree_large(siac_mod, oracle_mod, c, m, sch):
    """cfg 3 (graded) and cfg 4 (k = 4): the jump schedules against the oracle on a sample and
    against the clip-and-integrate schedule at every point."""
    w = cfg(c, "random")
    ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h)
    ctx.set_schedule(sch)
    gj = ctx.eval(w.points)
    ctx.set_schedule(2)
    gt = ctx.eval(w.points)
    ctx.destroy()
    assert_parity(gj, gt)
    idx = sample_idx(w.n_points, m, seed=100 + c)
    assert_parity(gj[idx], oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points[idx]))


@pytest.mark.parametrize("c,m", [(3, 1200), (4, 400), (5, 1500)])
def test_large_configs_sampled(siac_mod, oracle_mod, c, m):
    """All points on the GPU (bench launch configuration), oracle on a deterministic sample
    plus the points closest to the periodic boundary."""
    w = cfg(c)
    g = gpu_eval(siac_mod, w)
    idx = sample_idx(w.n_points, m, seed=c)
    edge = np.minimum.reduce([w.points[:, 0], 1 - w.points[:, 0], w.points[:, 1], 1 - w.points[:, 1]])
    idx = np.unique(np.concatenate([idx, np.argsort(edge)[:100]]))
    o = oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points[idx])
    assert_parity(g[idx], o)


def test_cfg5_random_field_sampled(siac_mod, oracle_mod):
    w = cfg(5, "random")
    g = gpu_eval(siac_mod, w)
    idx = sample_idx(w.n_points, 800, seed=55)
    assert_parity(g[idx], oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points[idx]))


# ------------------------------------------------------------------ invariants at full size

@pytest.mark.parametrize("c", [1, 2, 3, 4, 5])
def test_constant_field_every_point(siac_mod, c):
    """u = 1 -> u* = 1 at every point of every config (P3), any size."""
    w = cfg(c)
    C = np.zeros_like(w.C)
    C[:, 0] = math.sqrt(2.0)
    ctx = siac_mod.create(w.V, w.T, C, w.k, w.h)
    g = ctx.eval(w.points)
    ctx.destroy()
    assert np.abs(g - 1.0).max() < 1e-12


def test_deterministic_bitwise(siac_mod):
    w = cfg(3)
    ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h)
    a = ctx.eval(w.points)
    b = ctx.eval(w.points)
    ctx.destroy()
    assert np.array_equal(a, b)


def test_counters_agree_between_schedules(siac_mod):
    """The clip-and-integrate schedules clip the same pieces (pairs, pieces, sub-triangles
    agree); the jump schedule tests the same pairs and, at h = max edge, needs no general
    clipping: one corner term per pair and axis with a knot, cross terms only where both."""
    w = cfg(2)
    ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h)
    ctx.set_counting(True)
    got = []
    for sch in (2, 1, 3, 4, 5, 6):
        ctx.set_schedule(sch)
        ctx.eval(w.points)
        got.append(ctx.stats())
    ctx.destroy()
    s = got[0]
    assert s["n_points"] == w.n_points
    assert s["candidates"] >= s["pairs"] > 0
    assert s["subtris"] >= s["pieces"] >= s["pairs"] * 0.9
    for o in got[1:3]:
        assert got[0]["pairs"] == o["pairs"]
        assert abs(got[0]["pieces"] - o["pieces"]) <= 1e-4 * o["pieces"]
        assert abs(got[0]["subtris"] - o["subtris"]) <= 1e-4 * o["subtris"]
    j = got[3]
    assert j["pairs"] == s["pairs"] and j["pieces"] == 0 and j["subtris"] == 0
    # pieces per pair = (1 + [x knot]) (1 + [y knot]) summed, up to pieces outside the stencil
    assert 0 < j["cross_terms"] < j["corner_terms"] < 2 * j["pairs"]
    assert j["cross_subtris"] <= 2 * j["cross_terms"]
    assert j["pairs"] + j["corner_terms"] + j["cross_terms"] >= s["pieces"]
    x = got[4]      # closed-form cross terms: same pairs / corners / cross terms, no sub-triangles
    assert (x["pairs"], x["corner_terms"], x["cross_terms"]) == (j["pairs"], j["corner_terms"], j["cross_terms"])
    assert x["pieces"] == 0 and x["subtris"] == 0 and x["cross_subtris"] == 0
    assert 0 < x["cross_polys"] <= x["cross_terms"]
    e = got[5]      # per-element: the same pairs found from the other side (Eq. (3) element bounds)
    assert (e["pairs"], e["corner_terms"], e["cross_terms"], e["cross_polys"]) == \
        (x["pairs"], x["corner_terms"], x["cross_terms"], x["cross_polys"])
    assert e["candidates"] >= e["pairs"]


# ------------------------------------------------------------------ edge cases

EDGE_SCHEDULES = [0, 4, 6]     # default (JUMPX), JUMP, per-element


@pytest.mark.parametrize("sch", EDGE_SCHEDULES)
def test_random_points_anywhere_wrap(siac_mod, oracle_mod, sch):
    """Points outside [0,1)^2 wrap (periodic), including exact corners and edges."""
    w = cfg(2, "random")
    P = np.random.default_rng(1).uniform(-1.5, 2.5, (3000, 2))
    P[:6] = [[0, 0], [1, 1], [1, 0], [0.5, 1.0], [-1e-17, 0.3], [0.999999999999, 0.2]]
    assert_parity(gpu_eval(siac_mod, w, P, schedule=sch), oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, P))


@pytest.mark.parametrize("sch", EDGE_SCHEDULES)
@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_structured_breaklines_on_mesh_lines(siac_mod, oracle_mod, k, sch):
    """h = mesh spacing: kernel breaklines coincide with mesh lines (odd k) or mid-lines
    (even k); points at vertices, edge midpoints and cell centres; random field."""
    N = 16
    V, T = inputs.structured_mesh(N)
    C = inputs.random_modes(len(T), k, seed=k)
    h = 1.0 / N
    g1 = np.arange(0, N + 1) / N
    g2 = (np.arange(0, N) + 0.5) / N
    X = np.concatenate([g1, g2])
    P = np.array([[x, y] for x in X[::3] for y in X[::2]])
    ctx = siac_mod.create(V, T, C, k, h)
    ctx.set_schedule(sch)
    g = ctx.eval(P)
    ctx.destroy()
    assert_parity(g, oracle_mod.oracle_eval(V, T, C, k, h, P))


@pytest.mark.parametrize("sch", EDGE_SCHEDULES)
def test_stencil_equals_period(siac_mod, oracle_mod, sch):
    """W = (3k+1)h = period (k=1, N=4, h=1/4): every triangle meets the stencil through
    several periodic images (SURVEY A4 case)."""
    V, T = inputs.structured_mesh(4)
    C = inputs.random_modes(len(T), 1, seed=2)
    P = np.random.default_rng(3).uniform(0, 1, (200, 2))
    ctx = siac_mod.create(V, T, C, 1, 0.25)
    ctx.set_schedule(sch)
    g = ctx.eval(P)
    ctx.destroy()
    assert_parity(g, oracle_mod.oracle_eval(V, T, C, 1, 0.25, P))


@pytest.mark.parametrize("sch", EDGE_SCHEDULES)
def test_non_periodic_zero_extension(siac_mod, oracle_mod, sch):
    V, T = inputs.lattice_delaunay_mesh(3000, seed=9)
    k = 2
    C = inputs.random_modes(len(T), k, seed=4)
    h = inputs.max_edge(V, T)
    P = np.random.default_rng(5).uniform(-0.2, 1.2, (1500, 2))
    for per in (0, 1, 2):
        ctx = siac_mod.create(V, T, C, k, h, periodic=per)
        ctx.set_schedule(sch)
        g = ctx.eval(P)
        ctx.destroy()
        assert_parity(g, oracle_mod.oracle_eval(V, T, C, k, h, P, periodic=per))


@pytest.mark.parametrize("sch", EDGE_SCHEDULES)
def test_graded_small_h_and_large_h(siac_mod, oracle_mod, sch):
    """h other than the max edge: smaller (triangles span many kernel cells: the general
    clip-and-integrate path inside the jump schedules) and larger."""
    V, T = inputs.lattice_delaunay_mesh(2000, seed=12, graded=True)
    C = inputs.random_modes(len(T), 2, seed=6)
    P = inputs.eval_points(V, T, 2)[::17]
    for h in (0.25 * inputs.max_edge(V, T), 0.12):
        ctx = siac_mod.create(V, T, C, 2, h)
        ctx.set_schedule(sch)
        g = ctx.eval(P)
        ctx.destroy()
        assert_parity(g, oracle_mod.oracle_eval(V, T, C, 2, h, P))


@pytest.mark.parametrize("sch", EDGE_SCHEDULES)
def test_single_triangle_and_empty(siac_mod, oracle_mod, sch):
    V = np.array([[0.2, 0.3], [0.45, 0.31], [0.3, 0.5]])
    T = np.array([[0, 1, 2]], dtype=np.int32)
    C = inputs.random_modes(1, 3, seed=1)
    P = np.random.default_rng(2).uniform(0, 1, (257, 2))
    ctx = siac_mod.create(V, T, C, 3, 0.05, periodic=0)
    ctx.set_schedule(sch)
    assert ctx.eval(np.zeros((0, 2))).shape == (0,)
    g = ctx.eval(P)
    ctx.destroy()
    assert_parity(g, oracle_mod.oracle_eval(V, T, C, 3, 0.05, P, periodic=0))
    ctx0 = siac_mod.create(np.zeros((0, 2)), np.zeros((0, 3), np.int32), np.zeros((0, 3)), 1, 0.1)
    ctx0.set_schedule(sch)
    assert np.all(ctx0.eval(P) == 0.0)
    ctx0.destroy()


@pytest.mark.parametrize("sch", [0, 6])
@pytest.mark.parametrize("n", [1, 31, 32, 33, 1000, 4097])
def test_ragged_point_counts(siac_mod, oracle_mod, n, sch):
    w = cfg(2, "random")
    P = w.points[sample_idx(w.n_points, n, seed=n)]
    assert_parity(gpu_eval(siac_mod, w, P, schedule=sch), oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, P))


def test_async_torch_stream(siac_mod, oracle_mod):
    import torch
    w = cfg(1, "random")
    ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        P = torch.from_numpy(w.points).cuda()
        out = torch.empty(w.n_points, dtype=torch.float64, device="cuda")
        ctx.eval_async(P, out)
    s.synchronize()
    assert_parity(out.cpu().numpy(), oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points))
    ctx.destroy()


def test_cell_factor_invariance(siac_mod):
    """Results do not depend on the binning cell size (P10), bitwise up to summation order."""
    w = cfg(2, "random")
    outs = []
    for cf in (0.3, 0.5, 1.0, 2.0):
        outs.append(gpu_eval(siac_mod, w, cell_factor=cf))
    for o in outs[1:]:
        assert np.abs(o - outs[0]).max() <= 1e-12 * np.abs(outs[0]).max()


@pytest.mark.parametrize("sch", [0, 4, 6])
def test_graph_replay_matches_direct(siac_mod, sch):
    """siac_set_graphs: repeated eval_async on the same buffers replays a captured CUDA graph;
    results equal the direct path (bitwise, except the per-element schedule's atomics), across
    several buffer sets and after the scratch grows."""
    import torch
    w = cfg(2, "random")
    ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h)
    ctx.set_schedule(sch)
    s = torch.cuda.Stream()
    sets = []
    for n in (100, 1000, w.n_points):
        P = torch.from_numpy(np.ascontiguousarray(w.points[:n])).cuda()
        sets.append((P, torch.empty(n, dtype=torch.float64, device="cuda")))
    ref = [ctx.eval(P.cpu().numpy()) for P, _ in sets]
    ctx.set_graphs(True)
    with torch.cuda.stream(s):
        for rep in range(3):
            for (P, o), r in zip(sets, ref):
                o.fill_(np.nan)
                ctx.eval_async(P, o, s)
                s.synchronize()
                g = o.cpu().numpy()
                if sch == 6:
                    assert_parity(g, r, tol=1e-13)
                else:
                    assert np.array_equal(g, r)
    ctx.set_graphs(False)
    ctx.destroy()


# ------------------------------------------------------------------ full-size cross-checks (round 2)

def test_cfg5_jumpx_equals_tile_every_point(siac_mod):
    """Config 5 (1.05M triangles, P3, 12.6M points): the default schedule (JUMPX, spline-jump
    decomposition in closed form) against the direct clip-and-integrate schedule (TILE:
    Sutherland-Hodgman pieces, fan, degree-3k quadrature, Eq. (2) literally) at EVERY point,
    both in the bench's launch configuration.  Two unrelated decompositions of the same
    integral; the oracle pins the sample (test_large_configs_sampled)."""
    for field in ("sinsin", "random"):
        w = cfg(5, field)
        ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h)
        gj = ctx.eval(w.points)
        ctx.set_schedule(2)
        gt = ctx.eval(w.points)
        ctx.destroy()
        assert_parity(gj, gt)
        err = np.abs(gj - gt).max() / np.abs(gt).max()
        print(f"cfg5 {field}: JUMPX vs TILE normwise {err:.2e} over {w.n_points} points")
        assert err <= 1e-12


@pytest.mark.parametrize("c", [3, 5])
def test_partitioned_equals_single_gpu(siac_mod, c):
    """The multi-GPU split: for G = 2, 4, 8 ranks,
    dist.partition (Morton ranges of equal estimated work) + dist.local_problem (triangle halo)
    + one siac_create per partition, evaluated one after the other on this GPU and assembled,
    equals the single-context result at every point (only the summation grouping differs)."""
    from paper_conf_sc_0007k13_b200 import dist as sdist
    w = cfg(c, "random")
    ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h)
    ref = ctx.eval(w.points)
    ctx.destroy()
    hw = 0.5 * (3 * w.k + 1) * w.h
    wts = sdist.work_estimate(w.V, w.T, w.points, hw)
    for G in (2, 4, 8):
        part = sdist.partition(w.points, G, weights=wts)
        gathered = np.zeros((G, part["max_count"]))
        for r in range(G):
            loc = sdist.local_problem(w.V, w.T, w.C, w.points, w.k, w.h, part, r)
            assert len(loc["triangles"]) < len(w.T) or G == 2
            cr = siac_mod.create(loc["V"], loc["T"], loc["C"], w.k, w.h)
            gathered[r, :len(loc["points"])] = cr.eval(loc["points"])
            cr.destroy()
        got = sdist.assemble(gathered.ravel(), part, w.n_points)
        err = np.abs(got - ref).max() / np.abs(ref).max()
        print(f"cfg{c} G={G}: normwise {err:.2e}")
        assert err <= 1e-13


@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_monomial_ref_basis(siac_mod, oracle_mod, k):
    """params.basis = SIAC_BASIS_MONOMIAL_REF against the oracle's plain
    per-triangle monomial field (field_mode 2)."""
    V, T = inputs.lattice_delaunay_mesh(1500, seed=40 + k)
    M = np.random.default_rng(k).uniform(-1, 1, (len(T), inputs.n_modes(k)))
    h = inputs.max_edge(V, T)
    P = inputs.eval_points(V, T, k)[::7]
    ctx = siac_mod.create(V, T, M, k, h, basis=siac_mod.SIAC_BASIS_MONOMIAL_REF)
    g = ctx.eval(P)
    ctx.destroy()
    assert_parity(g, oracle_mod.oracle_eval(V, T, M, k, h, P, field_mode=2))


def test_create_info(siac_mod):
    """siac_get_create_info: stage times and the resident footprint of siac_create."""
    w = cfg(2)
    ctx = siac_mod.create(w.V, w.T, w.C, w.k, w.h)
    ci = ctx.create_info()
    ctx.destroy()
    for f in ("host_ms", "h2d_ms", "index_ms", "jump_ms", "cross_ms"):
        assert ci[f] >= 0.0
    assert ci["total_ms"] >= ci["h2d_ms"] + ci["index_ms"] + ci["jump_ms"] + ci["cross_ms"]
    assert ci["bytes_per_triangle"] > 8 * inputs.n_modes(w.k)
    assert ci["device_bytes"] >= ci["bytes_per_triangle"] * len(w.T)


# ------------------------------------------------------------------ one-sided kernels (NEXT-2)

def _onesided_tol(oracle_mod, k, h, P, periodic, domain=(0.0, 0.0, 1.0, 1.0)):
    """Per-point tolerance: north_star's 1e-10 relative, widened where the one-sided kernel's
    coefficients are large (rounding ~ eps (sum|c_x|)(sum|c_y|); reading R4)."""
    S = np.ones((len(P), 2))
    for ax in (0, 1):
        if not periodic & (1 << ax):
            lam = oracle_mod.onesided_shift(k, h, P[:, ax], domain[ax], domain[ax + 2])
            S[:, ax] = [sum(abs(float(c)) for c in oracle_mod.kernel_coefficients_shifted(k, float(l))) for l in lam]
    return 1e-15 * S[:, 0] * S[:, 1]


def _onesided_sample(V, T, k, h, periodic, m=240):
    """Element points: up to m inside the one-sided band of a non-periodic axis (every one has
    its own lambda; the oracle solves its moment system exactly per point), m/2 interior ones,
    plus the corners and edge midpoints."""
    P = inputs.eval_points(V, T, k)
    H = 0.5 * (3 * k + 1) * h
    band = np.zeros(len(P), dtype=bool)
    for ax in (0, 1):
        if not periodic & (1 << ax):
            band |= (P[:, ax] < H) | (P[:, ax] > 1 - H)
    rng = np.random.default_rng(k + 10 * periodic)
    bi, ii = np.nonzero(band)[0], np.nonzero(~band)[0]
    pick = np.concatenate([rng.choice(bi, min(m, len(bi)), replace=False),
                           rng.choice(ii, min(m // 2, len(ii)), replace=False)])
    extra = np.array([[0, 0], [1, 1], [0, 1], [1, 0], [0.5, 0], [0, 0.5], [1, 0.3], [0.7, 1]])
    return np.concatenate([P[np.sort(pick)], extra])


@pytest.mark.parametrize("k", [1, 2, 3, 4])
@pytest.mark.parametrize("periodic", [0, 1, 2])
def test_onesided_boundary_kernels(siac_mod, oracle_mod, k, periodic):
    """SIAC_BOUNDARY_ONESIDED (ref [21]) on a non-periodic Delaunay mesh
    covering the domain: every point, including boundary and corner points, against the
    oracle's per-point shifted-node kernels."""
    V, T = inputs.lattice_delaunay_mesh(3000, seed=50 + k)
    C = inputs.random_modes(len(T), k, seed=60 + k)
    h = inputs.max_edge(V, T)
    P = _onesided_sample(V, T, k, h, periodic)
    ctx = siac_mod.create(V, T, C, k, h, periodic=periodic, boundary=siac_mod.SIAC_BOUNDARY_ONESIDED)
    g = ctx.eval(P)
    ctx.destroy()
    o = oracle_mod.oracle_eval(V, T, C, k, h, P, periodic=periodic, boundary=1)
    tol = np.maximum(1e-10 * np.abs(o).max(), _onesided_tol(oracle_mod, k, h, P, periodic) * np.abs(o).max())
    assert np.all(np.abs(g - o) <= tol), f"max excess {np.max(np.abs(g - o) / tol):.3e}"
    assert_parity(g[np.abs(o) > 0], o[np.abs(o) > 0], tol=max(1e-10, float(_onesided_tol(oracle_mod, k, h, P, periodic).max())))


@pytest.mark.parametrize("k", [1, 3])
def test_onesided_reproduces_polynomials_to_the_boundary(siac_mod, k):
    """A global polynomial of degree k is reproduced at every point up to the corners (the
    one-sided kernel's purpose); zero extension is not (checked against the closed form)."""
    V, T = inputs.lattice_delaunay_mesh(4000, seed=70 + k)
    f = lambda x, y: 0.25 + (x - 0.4 * y) ** k - 0.6 * x * y ** (k - 1)  # noqa: E731
    C = inputs.project(V, T, k, f)
    h = inputs.max_edge(V, T)
    P = np.concatenate([inputs.eval_points(V, T, k)[::5], [[0, 0], [1, 1], [0, 1], [1, 0]]])
    ctx = siac_mod.create(V, T, C, k, h, periodic=0, boundary=siac_mod.SIAC_BOUNDARY_ONESIDED)
    g = ctx.eval(P)
    ctx.destroy()
    assert np.abs(g - f(P[:, 0], P[:, 1])).max() < 1e-9
    ctx = siac_mod.create(V, T, C, k, h, periodic=0)
    gz = ctx.eval(P)
    ctx.destroy()
    assert np.abs(gz - f(P[:, 0], P[:, 1])).max() > 1e-3


def test_onesided_small_h_general_path(siac_mod, oracle_mod):
    """h smaller than the triangles (the clip-and-integrate pass inside the jump schedule) with
    one-sided kernels on both axes."""
    V, T = inputs.lattice_delaunay_mesh(1500, seed=77, graded=True)
    k = 2
    C = inputs.random_modes(len(T), k, seed=78)
    h = 0.3 * inputs.max_edge(V, T)
    P = _onesided_sample(V, T, k, h, 0, m=200)
    ctx = siac_mod.create(V, T, C, k, h, periodic=0, boundary=1)
    g = ctx.eval(P)
    ctx.destroy()
    o = oracle_mod.oracle_eval(V, T, C, k, h, P, periodic=0, boundary=1)
    tol = np.maximum(1e-10, _onesided_tol(oracle_mod, k, h, P, 0)) * np.abs(o).max()
    assert np.all(np.abs(g - o) <= tol)


def test_onesided_rejects_other_schedules(siac_mod):
    V, T = inputs.lattice_delaunay_mesh(500, seed=1)
    C = inputs.random_modes(len(T), 1, seed=1)
    ctx = siac_mod.create(V, T, C, 1, inputs.max_edge(V, T), periodic=0, boundary=1)
    for sch in (1, 2, 3, 4, 6):
        ctx.set_schedule(sch)
        with pytest.raises(siac_mod.SiacError, match="one-sided|ONESIDED"):
            ctx.eval(np.array([[0.5, 0.5]]))
    ctx.destroy()
