#!/usr/bin/env python3
"""One 3D evaluation (siac3_eval_async, default schedule) for ncu captures:
python tools/profile3d.py NTET K [SCHEDULE]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    from paper_conf_sc_0007k13_b200 import siac
    from paper_conf_sc_0007k13_b200.inputs import mesh3d as m3
    ntet, k = int(sys.argv[1]), int(sys.argv[2])
    sch = int(sys.argv[3]) if len(sys.argv) > 3 else 0
    V, T = m3.lattice_delaunay_mesh3(ntet, seed=4000 + k)
    C = m3.project3(V, T, k, m3.sin3)
    h = min(m3.max_extent3(V, T), 0.95 / (3 * k + 1))
    P = m3.eval_points3(V, T)
    ctx = siac.create3(V, T, C, k, h)
    ctx.set_schedule(sch)
    d = torch.from_numpy(P).cuda()
    o = torch.empty(len(P), dtype=torch.float64, device="cuda")
    ctx.eval_async(d, o)
    torch.cuda.synchronize()
    print("ok", len(P), float(np.abs(o.cpu().numpy()).max()))
    ctx.destroy()


if __name__ == "__main__":
    main()
