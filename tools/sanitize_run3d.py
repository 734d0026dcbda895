"""A small tetrahedral evaluation for compute-sanitizer: both 3D schedules (0 = warp per tile with
the shared-memory piece queue and the split-tile combine, 1 = thread per point), k = 1 and 2, on a
Delaunay mesh small enough that tiles are split over several warps.
usage: compute-sanitizer --tool T python tools/sanitize_run3d.py"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    from paper_conf_sc_0007k13_b200 import siac
    from paper_conf_sc_0007k13_b200.inputs import mesh3d as m3
    for k in (1, 2):
        V, T = m3.lattice_delaunay_mesh3(400, seed=70 + k)
        C = m3.random_modes3(len(T), k, seed=80 + k)
        h = min(m3.max_extent3(V, T), 0.95 / (3 * k + 1))
        P = m3.eval_points3(V, T)[::3]
        vals = []
        for sch in (0, 1):
            ctx = siac.create3(V, T, C, k, h)
            ctx.set_schedule(sch)
            vals.append(ctx.eval(P))
            ctx.destroy()
        print(f"k={k} points={len(P)} schedules 0 vs 1 normwise {np.abs(vals[0] - vals[1]).max() / np.abs(vals[1]).max():.2e}")


if __name__ == "__main__":
    main()
