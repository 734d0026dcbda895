"""Multi-GPU host logic on CPU: partition, halo selection and the gather, with gloo as the
process group and the oracle as the per-rank evaluator (world_size 2 and 3)."""
import os
import socket

import numpy as np
import pytest

from paper_conf_sc_0007k13_b200 import dist as sdist
from paper_conf_sc_0007k13_b200 import inputs


def test_partition_covers_and_balances():
    w = inputs.make_config(2)
    for world in (1, 2, 3, 8):
        part = sdist.partition(w.points, world)
        assert part["bounds"][0] == 0 and part["bounds"][-1] == w.n_points
        assert np.array_equal(np.sort(part["order"]), np.arange(w.n_points))
        assert part["counts"].max() - part["counts"].min() <= 1
        assert part["max_count"] == part["counts"].max()


def test_partition_ranges_are_compact():
    """A quarter of the Morton curve is (up to a few boundary points) one quadrant."""
    w = inputs.make_config(2)
    part = sdist.partition(w.points, 4)
    for r in range(4):
        P = w.points[part["order"][part["bounds"][r]:part["bounds"][r + 1]]]
        lo, hi = np.quantile(P, 0.01, axis=0), np.quantile(P, 0.99, axis=0)
        assert (hi - lo).max() <= 0.55


def test_weighted_partition():
    P = np.random.default_rng(0).uniform(0, 1, (1000, 2))
    wts = np.where(P[:, 0] < 0.5, 3.0, 1.0)
    part = sdist.partition(P, 2, weights=wts)
    tot = [wts[part["order"][part["bounds"][r]:part["bounds"][r + 1]]].sum() for r in range(2)]
    assert abs(tot[0] - tot[1]) <= 3.0


@pytest.mark.parametrize("periodic", [3, 0])
def test_halo_contains_every_interacting_triangle(periodic):
    """Brute force: any triangle image whose box strictly overlaps a point's stencil square
    must be in the halo of that point's rank."""
    V, T = inputs.lattice_delaunay_mesh(1500, seed=3)
    k = 2
    h = inputs.max_edge(V, T)
    hw = 0.5 * (3 * k + 1) * h
    P = np.random.default_rng(1).uniform(0, 1, (400, 2))
    C = inputs.random_modes(len(T), k, seed=1)
    part = sdist.partition(P, 3, periodic=periodic)
    tx, ty = V[T][:, :, 0], V[T][:, :, 1]
    shifts = [(i, j) for i in ((-1, 0, 1) if periodic & 1 else (0,)) for j in ((-1, 0, 1) if periodic & 2 else (0,))]
    for r in range(3):
        loc = sdist.local_problem(V, T, C, P, k, h, part, r)
        have = set(loc["triangles"].tolist())
        for x in loc["points"]:
            for (i, j) in shifts:
                hit = ((tx.min(1) + i < x[0] + hw) & (tx.max(1) + i > x[0] - hw) &
                       (ty.min(1) + j < x[1] + hw) & (ty.max(1) + j > x[1] - hw))
                assert set(np.nonzero(hit)[0].tolist()) <= have

    # on a finer mesh with 8 ranks the halo is a proper subset
    V2, T2 = inputs.lattice_delaunay_mesh(16000, seed=4)
    h2 = inputs.max_edge(V2, T2)
    P2 = inputs.eval_points(V2, T2, 1)
    part2 = sdist.partition(P2, 8, periodic=periodic)
    loc = sdist.local_problem(V2, T2, inputs.random_modes(len(T2), 1, seed=2), P2, 1, h2, part2, 0)
    assert len(loc["triangles"]) < 0.5 * len(T2)


def test_assemble_inverts_partition():
    P = np.random.default_rng(2).uniform(0, 1, (101, 2))
    part = sdist.partition(P, 4)
    vals = np.arange(101, dtype=np.float64)
    g = np.zeros((4, part["max_count"]))
    for r in range(4):
        idx = part["order"][part["bounds"][r]:part["bounds"][r + 1]]
        g[r, :len(idx)] = vals[idx]
    assert np.array_equal(sdist.assemble(g.ravel(), part, 101), vals)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cfg, out_path):
    import torch.distributed as dist

    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    w = inputs.make_config(cfg, field_kind="random")

    def eval_fn(V, T, C, P):
        return oracle.oracle_eval(V, T, C, w.k, w.h, P, nthreads=2)

    got = sdist.dist_eval(w.V, w.T, w.C, w.points, w.k, w.h, eval_fn)
    if rank == 0:
        np.save(out_path, got)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_dist_eval_matches_single_process(world, tmp_path, oracle_mod):
    import torch.multiprocessing as mp
    out = str(tmp_path / "got.npy")
    mp.spawn(_worker, args=(world, _free_port(), 1, out), nprocs=world, join=True)
    got = np.load(out)
    w = inputs.make_config(1, field_kind="random")
    ref = oracle_mod.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points)
    assert np.abs(got - ref).max() <= 1e-13 * np.abs(ref).max()


def test_work_estimate_tracks_pair_counts_and_balances_graded_mesh():
    """The per-point work proxy follows the exact number of (point, triangle image) box pairs
    on the graded mesh (cfg 3), and partitioning by it balances the ranks' pairs where an
    equal-count partition does not."""
    w = inputs.make_config(3)
    hw = 0.5 * (3 * w.k + 1) * w.h
    est = sdist.work_estimate(w.V, w.T, w.points, hw)
    rng = np.random.default_rng(5)
    idx = rng.choice(w.n_points, 300, replace=False)
    tx, ty = w.V[w.T][:, :, 0], w.V[w.T][:, :, 1]
    exact = np.zeros(len(idx))
    for n, i in enumerate(idx):
        x = w.points[i]
        for a in (-1, 0, 1):
            for b in (-1, 0, 1):
                exact[n] += np.count_nonzero((tx.min(1) + a < x[0] + hw) & (tx.max(1) + a > x[0] - hw) &
                                             (ty.min(1) + b < x[1] + hw) & (ty.max(1) + b > x[1] - hw))
    assert exact.max() > 3 * exact.min()                       # the mesh is graded
    ratio = est[idx] / exact
    assert np.std(ratio) / np.mean(ratio) < 0.1                # proportional to the pair count
    world = 8          # (8 ranks: an equal-count cut is 2x out of balance on this mesh)
    spread = {}
    for name, wts in (("count", None), ("work", est)):
        part = sdist.partition(w.points, world, weights=wts)
        tot = [est[part["order"][part["bounds"][r]:part["bounds"][r + 1]]].sum() for r in range(world)]
        spread[name] = max(tot) / min(tot)
    assert spread["work"] < 1.01 and spread["count"] > 1.5


def _bcast_worker(rank, world, port, out_path):
    import torch
    import torch.distributed as dist

    import bench
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    w = inputs.make_config(2) if rank == 0 else None
    got, ms = bench.broadcast_workload(w, rank, torch.device("cpu"))
    if rank == 1:
        np.savez(out_path, V=got.V, T=got.T, C=got.C, P=got.points, k=got.k, h=got.h, n=got.n_points)
    dist.barrier()
    dist.destroy_process_group()


def test_bench_broadcasts_rank0_workload(tmp_path):
    """bench.py N > 1: rank 0 generates the workload once and broadcasts it;
    rank 1 receives bitwise the same mesh, modes and points (gloo, world 2)."""
    import torch.multiprocessing as mp
    out = str(tmp_path / "w.npz")
    mp.spawn(_bcast_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    got = np.load(out)
    w = inputs.make_config(2)
    for a, b in ((got["V"], w.V), (got["T"], w.T), (got["C"], w.C), (got["P"], w.points)):
        assert a.dtype == b.dtype and np.array_equal(a, b)
    assert int(got["k"]) == w.k and float(got["h"]) == w.h and int(got["n"]) == w.n_points


def test_near_cut_points_cover_halo_dependent_points():
    """dist.near_cut_points contains every point with a point of another rank inside its
    stencil square (brute force on a sample), and is a proper subset on a fine mesh."""
    w = inputs.make_config(3)
    hw = 0.5 * (3 * w.k + 1) * w.h
    part = sdist.partition(w.points, 8)
    near = set(sdist.near_cut_points(w.points, part, hw).tolist())
    owner = np.empty(w.n_points, dtype=np.int64)
    for r in range(8):
        owner[part["order"][part["bounds"][r]:part["bounds"][r + 1]]] = r
    rng = np.random.default_rng(3)
    for i in rng.choice(w.n_points, 400, replace=False):
        d = np.abs(w.points - w.points[i])
        d = np.minimum(d, 1 - d)
        if np.any((d.max(axis=1) < hw) & (owner != owner[i])):
            assert i in near
    assert len(sdist.near_cut_points(w.points, part, 0.02)) < 0.5 * w.n_points   # narrow stencil: a subset
