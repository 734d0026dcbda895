"""Debug: non-finite values per schedule, and non-finite entries of the device records."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_sc_0007k13_b200 import inputs, siac
c = int(sys.argv[1]) if len(sys.argv) > 1 else 2
w = inputs.make_config(c)
ctx = siac.create(w.V, w.T, w.C, w.k, w.h)
for sch in (4, 6, 0, 2):
    ctx.set_schedule(sch)
    v = ctx.eval(w.points)
    print(f"cfg{c} schedule {sch}: nonfinite {(~np.isfinite(v)).sum()} / {len(v)}", flush=True)
n = min(len(w.T), 2000)
for which in (0, 1, 2):
    r = ctx.debug_records(n, which)
    bad = ~np.isfinite(r)
    cols = np.nonzero(bad.any(0))[0]
    print(f"records {which}: shape {r.shape}, nonfinite {bad.sum()}, rows {bad.any(1).sum()}, cols {cols[:40].tolist()}")
    if which == 2:
        print("xrec[0][:8]", r[0, :8], "absmax", np.nanmax(np.abs(r[np.isfinite(r)])))
ctx.destroy()
