#!/usr/bin/env python3
"""Geometry counters of one evaluation: python tools/count_eval.py CFG [NPTS] [SCHEDULE]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_sc_0007k13_b200 import inputs, siac

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
npts = int(sys.argv[2]) if len(sys.argv) > 2 else 0
sch = int(sys.argv[3]) if len(sys.argv) > 3 else 0
w = inputs.make_config(cfg)
P = w.points[:npts] if npts else w.points
ctx = siac.create(w.V, w.T, w.C, w.k, w.h)
ctx.set_schedule(sch)
ctx.set_counting(True)
d = torch.from_numpy(np.ascontiguousarray(P)).cuda()
o = torch.empty(len(P), dtype=torch.float64, device="cuda")
ctx.eval_async(d, o)
s = ctx.stats()
print({k: (v / len(P) if k != "n_points" else v) for k, v in s.items()})
