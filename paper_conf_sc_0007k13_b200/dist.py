"""Multi-GPU SIAC evaluation: spatial point tiles per rank, triangle halos, NCCL gather.

PAPER.md §4/§5.2 (L641-645, L859-868) scale the per-element method by splitting the mesh
into N_GPU x N_SM patches with a two-stage reduction.  Here the evaluation points -- which
are independent ("outer parallelism where there is no inherent dependencies between grid
points", L862-864) -- are split instead, so no partial sums ever cross GPUs:

  partition()    points sorted along a Morton curve of the periodic domain and cut into
                 `world` contiguous, spatially compact ranges of equal estimated work
                 (work_estimate(): triangle centroids inside each point's stencil);
  halo()         each rank receives the triangles having a periodic image within the
                 stencil half-width W/2 = (3k+1)h/2 of its points (cell-dilation test);
  dist_eval()    siac_create on the halo subset, siac_eval_async on the rank's points, then
                 one all_gather_into_tensor of the padded per-rank values (8 B per point),
                 un-permuted into input order on every rank.

The evaluation itself is injected (`eval_fn`), so the same host logic runs on NCCL with the
CUDA library (bench.py) and on gloo with the oracle in CPU tests.  Host-side index bookkeeping
only: no part of the SIAC arithmetic lives here.
"""
from __future__ import annotations

import numpy as np


def _morton_keys(P, domain, bits=16):
    x0, y0, x1, y1 = domain
    n = (1 << bits) - 1
    ix = np.clip(((P[:, 0] - x0) / (x1 - x0) * n).astype(np.int64), 0, n)
    iy = np.clip(((P[:, 1] - y0) / (y1 - y0) * n).astype(np.int64), 0, n)

    def spread(v):
        v = (v | (v << 16)) & 0x0000FFFF0000FFFF
        v = (v | (v << 8)) & 0x00FF00FF00FF00FF
        v = (v | (v << 4)) & 0x0F0F0F0F0F0F0F0F
        v = (v | (v << 2)) & 0x3333333333333333
        v = (v | (v << 1)) & 0x5555555555555555
        return v

    return spread(ix) | (spread(iy) << 1)


def wrap_points(P, domain, periodic):
    P = np.array(P, dtype=np.float64, copy=True)
    x0, y0, x1, y1 = domain
    if periodic & 1:
        P[:, 0] = x0 + np.mod(P[:, 0] - x0, x1 - x0)
    if periodic & 2:
        P[:, 1] = y0 + np.mod(P[:, 1] - y0, y1 - y0)
    return P


def partition(points, world: int, domain=(0.0, 0.0, 1.0, 1.0), periodic: int = 3, weights=None) -> dict:
    """Split points into `world` Morton-contiguous ranges of equal total weight.

    weights: optional per-point work estimate (default 1 per point)."""
    P = wrap_points(points, domain, periodic)
    order = np.argsort(_morton_keys(P, domain), kind="stable")
    w = np.ones(len(P)) if weights is None else np.asarray(weights, dtype=np.float64)[order]
    cw = np.concatenate([[0.0], np.cumsum(w)])
    targets = cw[-1] * np.arange(1, world) / world
    cuts = np.searchsorted(cw, targets, side="left")
    bounds = np.concatenate([[0], cuts, [len(P)]]).astype(np.int64)
    counts = np.diff(bounds)
    return {"order": order, "bounds": bounds, "counts": counts, "max_count": int(max(counts.max(), 1)),
            "world": world, "domain": tuple(domain), "periodic": periodic}


def work_estimate(V, T, points, half_width, domain=(0.0, 0.0, 1.0, 1.0), periodic: int = 3) -> np.ndarray:
    """Per-point work proxy for partition(weights=...): the number of triangle centroids inside
    the point's stencil square (balance by estimated work, not point count; on
    graded meshes the pair count per point varies ~5x).  Centroids are binned on a grid of
    cells <= half_width / 4; a periodic-padded summed-area table gives each point's box count
    (the box rounded outward to whole cells, so it slightly over-counts uniformly)."""
    x0, y0, x1, y1 = domain
    Lx, Ly = x1 - x0, y1 - y0
    cen = V[T].mean(axis=1)
    nx = max(1, int(np.ceil(4 * Lx / half_width)))
    ny = max(1, int(np.ceil(4 * Ly / half_width)))
    cx, cy = Lx / nx, Ly / ny
    H, _, _ = np.histogram2d(np.clip((cen[:, 0] - x0) / cx, 0, nx - 1e-9), np.clip((cen[:, 1] - y0) / cy, 0, ny - 1e-9),
                             bins=[nx, ny], range=[[0, nx], [0, ny]])
    rx, ry = int(np.ceil(half_width / cx)) + 1, int(np.ceil(half_width / cy)) + 1
    Hp = np.pad(H, ((rx, rx), (ry, ry)), mode="wrap" if periodic == 3 else "constant")
    if periodic in (1, 2):
        Hp = np.pad(H, ((rx, rx), (0, 0)), mode="wrap" if periodic & 1 else "constant")
        Hp = np.pad(Hp, ((0, 0), (ry, ry)), mode="wrap" if periodic & 2 else "constant")
    S = np.zeros((Hp.shape[0] + 1, Hp.shape[1] + 1))
    S[1:, 1:] = Hp.cumsum(0).cumsum(1)
    P = wrap_points(points, domain, periodic)
    i0 = np.floor((P[:, 0] - half_width - x0) / cx).astype(np.int64) + rx
    i1 = np.floor((P[:, 0] + half_width - x0) / cx).astype(np.int64) + rx + 1
    j0 = np.floor((P[:, 1] - half_width - y0) / cy).astype(np.int64) + ry
    j1 = np.floor((P[:, 1] + half_width - y0) / cy).astype(np.int64) + ry + 1
    i0, i1 = np.clip(i0, 0, Hp.shape[0]), np.clip(i1, 0, Hp.shape[0])
    j0, j1 = np.clip(j0, 0, Hp.shape[1]), np.clip(j1, 0, Hp.shape[1])
    return S[i1, j1] - S[i0, j1] - S[i1, j0] + S[i0, j0]


def halo(V, T, points, half_width, domain=(0.0, 0.0, 1.0, 1.0), periodic: int = 3) -> np.ndarray:
    """Indices (ascending) of every triangle that has a periodic image within half_width of
    some point's stencil centre box, i.e. every triangle that can meet a stencil.

    Conservative cell test: points mark the cells of a uniform grid (cell >= the largest
    triangle extent), the marks are dilated by ceil(half_width / cell) + 1 cells (wrapping on
    periodic axes), and a triangle is kept if a cell under its bounding box is marked."""
    from scipy.ndimage import maximum_filter

    x0, y0, x1, y1 = domain
    Lx, Ly = x1 - x0, y1 - y0
    tx, ty = V[T][:, :, 0], V[T][:, :, 1]
    ext = max(float((tx.max(1) - tx.min(1)).max(initial=0.0)), float((ty.max(1) - ty.min(1)).max(initial=0.0)))
    c = max(ext, half_width / 64.0, 1e-9 * max(Lx, Ly))
    nx, ny = max(1, int(Lx / c)), max(1, int(Ly / c))
    cx, cy = Lx / nx, Ly / ny
    P = wrap_points(points, domain, periodic)
    mark = np.zeros((ny, nx), dtype=np.uint8)
    pi = np.clip(((P[:, 0] - x0) / cx).astype(np.int64), 0, nx - 1)
    pj = np.clip(((P[:, 1] - y0) / cy).astype(np.int64), 0, ny - 1)
    mark[pj, pi] = 1
    rx, ry = int(np.ceil(half_width / cx)) + 1, int(np.ceil(half_width / cy)) + 1
    if (periodic & 1 and 2 * rx + 1 >= nx) or (periodic & 2 and 2 * ry + 1 >= ny):
        return np.arange(len(T))
    mark = maximum_filter(mark, size=(1, 2 * rx + 1), mode="wrap" if periodic & 1 else "constant")
    mark = maximum_filter(mark, size=(2 * ry + 1, 1), mode="wrap" if periodic & 2 else "constant")
    i0 = np.clip(np.floor((tx.min(1) - x0) / cx).astype(np.int64), 0, nx - 1)
    i1 = np.clip(np.floor((tx.max(1) - x0) / cx).astype(np.int64), 0, nx - 1)
    j0 = np.clip(np.floor((ty.min(1) - y0) / cy).astype(np.int64), 0, ny - 1)
    j1 = np.clip(np.floor((ty.max(1) - y0) / cy).astype(np.int64), 0, ny - 1)
    keep = (mark[j0, i0] | mark[j0, i1] | mark[j1, i0] | mark[j1, i1]).astype(bool)
    return np.nonzero(keep)[0]


def near_cut_points(points, part: dict, half_width: float) -> np.ndarray:
    """Indices (ascending) of the points whose stencil square (half-width `half_width`) reaches
    a cell holding points of another rank: the points whose values depend on the halo
    (parity "plus points within W of partition boundaries").  Cell test on a
    grid of cells >= half_width, wrapping on periodic axes; conservative."""
    x0, y0, x1, y1 = part["domain"]
    periodic = part["periodic"]
    P = wrap_points(points, part["domain"], periodic)
    nx = max(1, int((x1 - x0) / half_width))
    ny = max(1, int((y1 - y0) / half_width))
    ix = np.clip(((P[:, 0] - x0) / (x1 - x0) * nx).astype(np.int64), 0, nx - 1)
    iy = np.clip(((P[:, 1] - y0) / (y1 - y0) * ny).astype(np.int64), 0, ny - 1)
    owner = np.empty(len(P), dtype=np.int64)
    for r in range(part["world"]):
        owner[part["order"][part["bounds"][r]:part["bounds"][r + 1]]] = r
    lo = np.full((ny, nx), part["world"], dtype=np.int64)
    hi = np.full((ny, nx), -1, dtype=np.int64)
    np.minimum.at(lo, (iy, ix), owner)
    np.maximum.at(hi, (iy, ix), owner)
    near = np.zeros(len(P), dtype=bool)
    for dj in (-1, 0, 1):
        for di in (-1, 0, 1):
            jj, ii = iy + dj, ix + di
            ok = np.ones(len(P), dtype=bool)
            if periodic & 1:
                ii = ii % nx
            else:
                ok &= (ii >= 0) & (ii < nx)
            if periodic & 2:
                jj = jj % ny
            else:
                ok &= (jj >= 0) & (jj < ny)
            jj, ii = np.clip(jj, 0, ny - 1), np.clip(ii, 0, nx - 1)
            other = ok & (((lo[jj, ii] != owner) & (lo[jj, ii] < part["world"])) | ((hi[jj, ii] != owner) & (hi[jj, ii] >= 0)))
            near |= other
    return np.nonzero(near)[0]


def local_problem(V, T, C, points, k: int, h: float, part: dict, rank: int) -> dict:
    """The rank's points (in partition order) and its halo triangles."""
    lo, hi = part["bounds"][rank], part["bounds"][rank + 1]
    idx = part["order"][lo:hi]
    P = np.asarray(points, dtype=np.float64)[idx]
    if len(P):
        sel = halo(V, T, P, 0.5 * (3 * k + 1) * h, part["domain"], part["periodic"])
    else:
        sel = np.zeros(0, dtype=np.int64)
    return {"V": V, "T": np.ascontiguousarray(T[sel]), "C": np.ascontiguousarray(C[sel]), "points": P,
            "point_index": idx, "triangles": sel}


def assemble(gathered, part: dict, n_points: int) -> np.ndarray:
    """Padded per-rank slices (world x max_count, partition order) -> values in input order."""
    out = np.empty(n_points, dtype=np.float64)
    g = np.asarray(gathered).reshape(part["world"], part["max_count"])
    for r in range(part["world"]):
        lo, hi = part["bounds"][r], part["bounds"][r + 1]
        out[part["order"][lo:hi]] = g[r, : hi - lo]
    return out


def dist_eval(V, T, C, points, k: int, h: float, eval_fn, group=None, periodic: int = 3,
              domain=(0.0, 0.0, 1.0, 1.0), device=None, balance: str = "work"):
    """Evaluate u* at all points over the ranks of `group` (torch.distributed); every rank
    returns the full result in input order.

    eval_fn(V, T, C, points_local) -> values_local (numpy or torch tensor on `device`)."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    wts = work_estimate(V, T, points, 0.5 * (3 * k + 1) * h, domain, periodic) if balance == "work" else None
    part = partition(points, world, domain, periodic, weights=wts)
    loc = local_problem(V, T, C, points, k, h, part, rank)
    vals = eval_fn(loc["V"], loc["T"], loc["C"], loc["points"])
    dev = device if device is not None else torch.device("cpu")
    send = torch.zeros(part["max_count"], dtype=torch.float64, device=dev)
    v = torch.as_tensor(vals, dtype=torch.float64, device=dev)
    send[: len(v)] = v
    recv = torch.empty(world * part["max_count"], dtype=torch.float64, device=dev)
    dist.all_gather_into_tensor(recv, send, group=group)
    return assemble(recv.cpu().numpy(), part, len(points))
