#!/usr/bin/env python3
"""NEXT-4 measurement: filtered points/s of the tetrahedral path (siac3_eval_async, inputs
resident in HBM, CUDA events; W >= 3 warm-ups), its geometry counts, a model FP64 rate, and
parity against the 3D oracle on a sample.  Not the driver's bench (the north_star metric is
2D); results go to profiles/.

Both mappings are timed: schedule 0 (warp per point tile, default) and 1 (thread per point).

usage: python tools/bench3d.py [ntet] [k] [steps] [oracle_points] [out.json] [time_schedule_1]
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import oracle
    from bench import parity_report
    from paper_conf_sc_0007k13_b200 import siac
    from paper_conf_sc_0007k13_b200.inputs import mesh3d as m3

    ntet = int(sys.argv[1]) if len(sys.argv) > 1 else 8000
    k = int(sys.argv[2]) if len(sys.argv) > 2 else 1
    steps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
    nor = int(sys.argv[4]) if len(sys.argv) > 4 else 24
    out_path = sys.argv[5] if len(sys.argv) > 5 else None
    tpp = int(sys.argv[6]) if len(sys.argv) > 6 else 1      # also time schedule 1 (thread per point)
    V, T = m3.lattice_delaunay_mesh3(ntet, seed=4000 + k)
    C = m3.project3(V, T, k, m3.sin3)
    h = min(m3.max_extent3(V, T), 0.95 / (3 * k + 1))     # W = (3k+1)h must fit the period
    P = m3.eval_points3(V, T)
    t0 = time.perf_counter()
    ctx = siac.create3(V, T, C, k, h)
    create_ms = 1e3 * (time.perf_counter() - t0)
    d = torch.from_numpy(P).cuda()
    o = torch.empty(len(P), dtype=torch.float64, device="cuda")

    def timed(schedule):
        ctx.set_schedule(schedule)
        ctx.set_counting(True)
        ctx.eval_async(d, o)
        st = ctx.stats()
        ctx.set_counting(False)
        for _ in range(3):
            ctx.eval_async(d, o)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(steps):
            ctx.eval_async(d, o)
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / steps, st, o.cpu().numpy()

    ms, st, g = timed(0)             # warp per point tile (default)
    ms1, st1, g1 = timed(1) if tpp else (None, None, None)   # thread per point (the paper's per-point mapping)
    ctx.destroy()
    nq = (2 * k + 1) ** 3
    nb = m3.n_modes3(k)
    # model flops per quadrature point: map to z (9 FMA), three degree-k Horners (3k FMA), affine
    # map to (r, s, t) (9 FMA), the monomial sum (nb FMA + powers 3(k-1) mul), product/weight (3);
    # an FMA counts 2; plus ~30 per piece (edges, volume)
    f_qp = 2 * (9 + 3 * k + 9 + nb + 3) + 3 * (k - 1)
    flops = st["pieces"] * (nq * f_qp + 30)
    peak = 148 * 64 * 2 * 1965e6
    idx = np.linspace(0, len(P) - 1, nor).astype(np.int64)
    t0 = time.perf_counter()
    ref = oracle.oracle_eval3(V, T, C, k, h, P[idx], nthreads=oracle.omp_threads())
    ot = time.perf_counter() - t0
    res = {"what": "NEXT-4 tetrahedral path (siac3_eval_async), FP64", "n_tets": int(len(T)), "n_points": int(len(P)),
           "k": k, "h": h, "mesh": "jittered-lattice Delaunay (scipy), periodic unit cube", "field": "sin sin sin, L2",
           "schedule": "0: warp per 32-point tile, pieces queued in shared memory, quadrature in lock step",
           "ms_per_eval": ms, "points_per_s": len(P) / (ms * 1e-3), "create_ms": create_ms,
           "thread_per_point": None if not tpp else {"schedule": 1, "ms_per_eval": ms1, "points_per_s": len(P) / (ms1 * 1e-3),
                                "model_frac_of_fp64_peak": flops / (ms1 * 1e-3) / peak,
                                "same_counts": st1 == st,
                                "max_rel_diff_vs_schedule0": float(np.abs(g1 - g).max() / np.abs(g).max())},
           "pairs": st["pairs"], "pieces": st["pieces"], "pairs_per_point": st["pairs"] / len(P),
           "pieces_per_pair": st["pieces"] / max(st["pairs"], 1), "quadrature_points_per_piece": nq,
           "model_flops_per_eval": flops, "model_tflops": flops / (ms * 1e-3) / 1e12,
           "model_frac_of_fp64_peak": flops / (ms * 1e-3) / peak,
           "parity": dict(parity_report(g[idx], ref), sample=f"{nor} evenly spaced points"),
           "oracle_points_per_s": nor / ot, "oracle_cores": oracle.omp_threads(),
           "gpu": torch.cuda.get_device_name(0)}
    print(json.dumps(res, indent=1))
    if out_path:
        with open(out_path, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
