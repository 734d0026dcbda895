#!/usr/bin/env python3
"""the paper's per-point vs per-element comparison on B200.

Table 1 analogue: intersection tests (bounding-box candidate tests) of the
per-point search (schedule POINT: cell c_p = s, halo cells around the stencil, Eq. (3) per-point
bounds) and of the per-element search (schedule ELEM: cell c_e = s/2, Eq. (3) per-element
bounds), P1 with 3 points per element, on the synthetic jittered-lattice Delaunay meshes of
~4k..1024k triangles (the paper's meshes are not available).  Fig. 13 analogue: evaluation time
of the per-point direct method (POINT, Alg. 2: thread per point, SH clip + fan + quadrature),
the per-element schedule (ELEM, Alg. 3 mapping) and the point-tile jump schedule (JUMPX) for
P = 1, 2, 3.

usage (GPU): python tools/table1.py OUT.json [max_ntri]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_sc_0007k13_b200 import inputs, siac

PAPER_TABLE1 = {  # PAPER.md Table 1 (L516-536): mesh size -> (per-point, per-element) tests, P1
    "4k": (6647394, 3525297), "16k": (26492809, 14235618), "64k": (110778427, 59277119),
    "256k": (455614318, 243245703), "1024k": (1919070326, 1017924543)}


def timed(ctx, d, o, reps=2):
    ctx.eval_async(d, o)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        ctx.eval_async(d, o)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def counts(V, T, C, k, h, P, sched, cf):
    ctx = siac.create(V, T, C, k, h, cell_factor=cf)
    ctx.set_schedule(sched)
    ctx.set_counting(True)
    d = torch.from_numpy(np.ascontiguousarray(P)).cuda()
    o = torch.empty(len(P), dtype=torch.float64, device="cuda")
    ctx.eval_async(d, o)
    st = ctx.stats()
    ctx.destroy()
    return st


def main():
    out_path = sys.argv[1]
    max_nt = int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 20
    res = {"table1": [], "fig13": [], "note": __doc__}
    for j, (label, ntri) in enumerate([("4k", 4096), ("16k", 16384), ("64k", 65536), ("256k", 262144),
                                        ("1024k", 1048576)]):
        if ntri > max_nt:
            break
        V, T = inputs.lattice_delaunay_mesh(ntri, 3000 + j)
        h = inputs.max_edge(V, T)
        for k in (1, 2, 3):
            C = inputs.random_modes(len(T), k, 11 + k)
            P = inputs.eval_points(V, T, k)
            if k == 1:
                pp = counts(V, T, C, k, h, P, 1, 1.0)        # per-point: c_p = s
                pe = counts(V, T, C, k, h, P, 6, 0.5)        # per-element: c_e = s/2
                row = {"mesh": label, "ntri": len(T), "npts": len(P), "h": h,
                       "per_point_tests": pp["candidates"], "per_element_tests": pe["candidates"],
                       "ratio": pp["candidates"] / max(pe["candidates"], 1), "pairs": pe["pairs"],
                       "paper_per_point": PAPER_TABLE1[label][0], "paper_per_element": PAPER_TABLE1[label][1],
                       "paper_ratio": PAPER_TABLE1[label][0] / PAPER_TABLE1[label][1]}
                res["table1"].append(row)
                print(json.dumps(row), flush=True)
            d = torch.from_numpy(np.ascontiguousarray(P)).cuda()
            o = torch.empty(len(P), dtype=torch.float64, device="cuda")
            row = {"mesh": label, "ntri": len(T), "k": k, "npts": len(P)}
            vals = {}
            for name, sched in (("per_point_direct", 1), ("per_element", 6), ("point_tile_jumpx", 5)):
                ctx = siac.create(V, T, C, k, h)
                ctx.set_schedule(sched)
                row[name + "_ms"] = timed(ctx, d, o, reps=1 if sched == 1 and len(P) > 2e6 else 2)
                vals[name] = o.cpu().numpy()
                ctx.destroy()
            ref = vals["point_tile_jumpx"]
            row["max_rel_diff"] = max(float(np.abs(v - ref).max() / np.abs(ref).max()) for v in vals.values())
            res["fig13"].append(row)
            print(json.dumps(row), flush=True)
    json.dump(res, open(out_path, "w"), indent=1)


if __name__ == "__main__":
    main()
