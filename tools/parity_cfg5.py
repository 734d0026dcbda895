"""Survey-sized parity run at the benchmarked configuration (SURVEY §8(d) "Oracle timing"):
config 5 evaluated completely on the GPU in the bench's launch configuration (siac_eval_async,
default schedule), the oracle on a 1/128 deterministic stride subset plus 4,096 points within
the stencil half-width of the 8-way partition cuts (points whose values depend on the halos),
and parity on exactly those points.

usage: python tools/parity_cfg5.py [field] [out.json]      (field: sinsin | random)
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
    from paper_conf_sc_0007k13_b200 import dist as sdist
    from paper_conf_sc_0007k13_b200 import inputs, siac

    field = sys.argv[1] if len(sys.argv) > 1 else "sinsin"
    out_path = sys.argv[2] if len(sys.argv) > 2 else None
    w = inputs.make_config(5, field_kind=field)
    ctx = siac.create(w.V, w.T, w.C, w.k, w.h)
    d_pts = torch.from_numpy(w.points).cuda()
    d_out = torch.empty(w.n_points, dtype=torch.float64, device="cuda")
    ctx.eval_async(d_pts, d_out)
    torch.cuda.synchronize()
    g = d_out.cpu().numpy()
    ctx.destroy()
    hw = 0.5 * (3 * w.k + 1) * w.h
    part = sdist.partition(w.points, 8, weights=sdist.work_estimate(w.V, w.T, w.points, hw))
    near = sdist.near_cut_points(w.points, part, hw)
    rng = np.random.default_rng(128)
    pick = np.sort(rng.choice(near, size=min(4096, len(near)), replace=False))
    stride = np.arange(0, w.n_points, 128)
    idx = np.unique(np.concatenate([stride, pick]))
    t0 = time.perf_counter()
    o = oracle.oracle_eval(w.V, w.T, w.C, w.k, w.h, w.points[idx], nthreads=oracle.omp_threads())
    dt = time.perf_counter() - t0
    rep = parity_report(g[idx], o)
    rep_cut = parity_report(g[pick], o[np.searchsorted(idx, pick)])
    res = {"config": 5, "field": field, "n_points": int(w.n_points), "n_triangles": int(len(w.T)),
           "sample": {"stride": 128, "stride_points": int(len(stride)), "near_cut_points": int(len(pick)),
                      "near_cut_pool": int(len(near)), "total": int(len(idx))},
           "parity": rep, "parity_near_cuts": rep_cut,
           "oracle_seconds": dt, "oracle_cores": oracle.omp_threads(),
           "gpu": torch.cuda.get_device_name(0), "schedule": "default (JUMPX)"}
    print(json.dumps(res, indent=1))
    if out_path:
        with open(out_path, "w") as f:
            json.dump(res, f, indent=1)
    assert rep["pass"] and rep_cut["pass"]


if __name__ == "__main__":
    main()
