#!/usr/bin/env python3
"""Run k_eval on a workload subset for profiling (ncu / sanitizer): python tools/profile_eval.py CFG NPTS REPS"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_sc_0007k13_b200 import inputs, siac

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
npts = int(sys.argv[2]) if len(sys.argv) > 2 else 200000
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
w = inputs.make_config(cfg)
P = w.points
if npts < len(P):
    # a spatially contiguous block of elements (like one GPU's tile of the domain)
    P = P[:npts]
ctx = siac.create(w.V, w.T, w.C, w.k, w.h)
d = torch.from_numpy(np.ascontiguousarray(P)).cuda()
o = torch.empty(len(P), dtype=torch.float64, device="cuda")
for _ in range(reps):
    ctx.eval_async(d, o)
torch.cuda.synchronize()
print("done", len(P), float(o[:4].sum()))
