#!/usr/bin/env python3
"""Quick A/B timing of the evaluation kernel: python tools/quick_time.py [cfg ...] (default 2 3 5)
Prints ms per eval (CUDA events) for each schedule and a parity spot check between them."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_sc_0007k13_b200 import inputs, siac

cfgs = [int(c) for c in sys.argv[1:]] or [2, 3, 5]
for c in cfgs:
    w = inputs.make_config(c)
    P = w.points if (c != 5 or os.environ.get("QT_FULL")) else w.points[: 2_000_000]
    ctx = siac.create(w.V, w.T, w.C, w.k, w.h)
    d = torch.from_numpy(np.ascontiguousarray(P)).cuda()
    outs = {}
    for sch in [int(x) for x in os.environ.get("QT_SCHED", "0,2").split(",")]:
        ctx.set_schedule(sch)
        o = torch.empty(len(P), dtype=torch.float64, device="cuda")
        ctx.eval_async(d, o)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 3
        e0.record()
        for _ in range(reps):
            ctx.eval_async(d, o)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        outs[sch] = o.cpu().numpy()
        print(f"cfg{c} sched={sch} npts={len(P)} {ms:9.2f} ms  {len(P) / ms * 1e3:12.0f} pts/s", flush=True)
    ks = list(outs); diff = np.abs(outs[ks[0]] - outs[ks[-1]]).max() / np.abs(outs[ks[-1]]).max()
    print(f"cfg{c} first vs last schedule normwise diff {diff:.2e}", flush=True)
    ctx.destroy()
