#!/usr/bin/env python3
"""Run the evaluation on a workload subset for profiling (ncu / sanitizer):
    python tools/profile_eval.py CFG NPTS REPS [SCHEDULE]
The subset is the NPTS points nearest the domain centre (a spatially compact block, like one
GPU's share of a Morton-ordered run), so caches see the same locality as the full run."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_sc_0007k13_b200 import inputs, siac

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
npts = int(sys.argv[2]) if len(sys.argv) > 2 else 200000
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
sch = int(sys.argv[4]) if len(sys.argv) > 4 else 0
w = inputs.make_config(cfg)
P = w.points
if npts < len(P):
    d = np.max(np.abs(P - 0.5), axis=1)          # square window around the centre
    P = P[np.argsort(d, kind="stable")[:npts]]
ctx = siac.create(w.V, w.T, w.C, w.k, w.h)
ctx.set_schedule(sch)
d = torch.from_numpy(np.ascontiguousarray(P)).cuda()
o = torch.empty(len(P), dtype=torch.float64, device="cuda")
for _ in range(reps):
    ctx.eval_async(d, o)
torch.cuda.synchronize()
print("done", len(P), float(o[:4].sum()))
