#!/usr/bin/env python3
"""Per-call time of small repeated evaluations with and without CUDA-graph replay (siac_set_graphs)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_sc_0007k13_b200 import inputs, siac
for c in (1, 2):
    w = inputs.make_config(c)
    ctx = siac.create(w.V, w.T, w.C, w.k, w.h)
    s = torch.cuda.Stream()
    P = torch.from_numpy(w.points).cuda(); o = torch.empty(w.n_points, dtype=torch.float64, device='cuda')
    for graphs in (False, True):
        ctx.set_graphs(graphs)
        with torch.cuda.stream(s):
            for _ in range(5): ctx.eval_async(P, o, s)
            s.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s); 
            for _ in range(200): ctx.eval_async(P, o, s)
            e1.record(s); s.synchronize()
        print(f"cfg{c} graphs={graphs} {e0.elapsed_time(e1)/200*1e3:.1f} us per eval", flush=True)
    ctx.destroy()
