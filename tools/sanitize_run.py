"""Small evaluations for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).

usage: compute-sanitizer --tool T python tools/sanitize_run.py CFG SCHEDULES [graphs]

Runs siac_create + siac_eval (host buffers) and siac_eval_async on a torch stream for each
listed schedule on BASELINE config CFG (1 or 2: the small configs, where the split-warp
partial-sum path of the jump schedules is active because there are fewer point tiles than
resident warps).  With "graphs", the async evaluation is also captured as a CUDA graph and
replayed (siac_set_graphs).  Prints the normwise difference between schedules so a run that
"passes" the sanitizer while computing garbage is visible.
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    from paper_conf_sc_0007k13_b200 import inputs, siac

    cfg = int(sys.argv[1])
    schedules = [int(s) for s in sys.argv[2].split(",")]
    graphs = len(sys.argv) > 3 and sys.argv[3] == "graphs"
    w = inputs.make_config(cfg, field_kind="random")
    ctx = siac.create(w.V, w.T, w.C, w.k, w.h, periodic=3)
    ref = None
    st = torch.cuda.Stream()
    d_pts = torch.from_numpy(w.points).cuda()
    d_out = torch.empty(w.n_points, dtype=torch.float64, device="cuda")
    for sch in schedules:
        ctx.set_schedule(sch)
        v = ctx.eval(w.points)
        with torch.cuda.stream(st):
            ctx.eval_async(d_pts, d_out, st)
        st.synchronize()
        va = d_out.cpu().numpy()
        if graphs:
            ctx.set_graphs(True)
            for _ in range(3):
                ctx.eval_async(d_pts, d_out, st)
            st.synchronize()
            vg = d_out.cpu().numpy()
            ctx.set_graphs(False)
            assert np.array_equal(vg, va) or sch == 6, "graph replay differs"
        ref = v if ref is None else ref
        err = np.abs(v - ref).max() / np.abs(ref).max()
        erra = np.abs(va - v).max() / np.abs(v).max()
        print(f"cfg{cfg} schedule {sch}: {w.n_points} points, vs first {err:.2e}, async vs sync {erra:.2e}"
              + (" graphs ok" if graphs else ""), flush=True)
        assert err < 1e-10 and erra < 1e-10
    ctx.set_counting(True)
    ctx.eval(w.points)
    print("counters", ctx.stats(), flush=True)
    ctx.destroy()
    print("done", flush=True)


if __name__ == "__main__":
    main()
