#!/usr/bin/env python3
"""bench.py -- filtered quadrature points/s (FP64) of the B200 SIAC path.

Contract (driver): `python bench.py --gpus N --steps K --warmup W` (torchrun for N > 1)
prints ONE JSON line on rank 0.  A step = one siac_eval_async over every evaluation point of
the workload (all §8(a) rows: point keys + sort, candidate search, clipping, fan
triangulation, quadrature, per-point reduction), inputs resident in HBM.  Default workload:
BASELINE.json config 5 (Delaunay ~1M triangles, P3, 12 points/element = 12.6M points), the
configuration the metric is quoted on at 1/2/4/8 GPUs; it fits one GPU.

`--impl reference` times the oracle (the CPU reference arm of this tier) on a bounded
sample of the same workload.
"""
import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# quadrature points per sub-triangle and FP64 flops per quadrature point:
# F_qp = 2 (n_b + 2k + 8)  (affine map 4, two degree-k Horner 2k, frame offsets 2,
# bivariate Horner n_b - 1, product/weight/accumulate 3; an FMA counts 2 flops)
NQ = {1: 4, 2: 12, 3: 19, 4: 33}


def flops_per_subtri(k):
    nb = (k + 1) * (k + 2) // 2
    return NQ[k] * 2 * (nb + 2 * k + 8)


# Schedules JUMP / JUMPX (JUMPX is the default) compute the same integral through the spline-jump decomposition
# (DESIGN.md §8.2); its algorithmic FP64 flops per unit, counted from the operations the
# decomposition needs (an FMA counts 2):
#   per (point, triangle) pair: two cut tests (10 each), two Taylor shifts of the base cell
#     polynomials (K(K+1)/2 FMA each) and the moment contraction ((K+1)^2 + (K+1) FMA);
#   per corner term: the G contraction (NG FMA), the Horner pass in lambda (2K FMA), the
#     lambda^(K+2) power (K+1 mul) and the accumulate (1 FMA);
#   per cross sub-triangle (schedule 4): NQ quadrature points x (affine maps 8 FMA, bivariate
#     Horner NB-1 FMA, product/weight 2 FMA, t^K: K mul) + 20 set-up;
#   per interval-polynomial cross term (schedule 5, default): a bivariate Horner/Estrin pass over
#     NP = (K+1)(3K+3) monomial coefficients (1 FMA each) + lambda^(2K+2) and the mapping (~2K + 12).
def jump_flops(k, pairs, corners, cross_subtris, cross_polys=0):
    nb = (k + 1) * (k + 2) // 2
    ng = (k + 1) * (3 * k + 2) // 2
    npoly = (k + 1) * (3 * k + 3)
    f_pair = 20 + 2 * (k * (k + 1) + (k + 1) * (k + 2))
    f_corner = 2 * (ng + 2 * k + 1) + (k + 1)
    f_xsub = NQ[k] * (2 * (nb + 9) + k) + 20
    f_xpoly = 2 * npoly + 2 * k + 12
    return (pairs * f_pair + corners * f_corner + cross_subtris * f_xsub + cross_polys * f_xpoly,
            (f_pair, f_corner, f_xsub, f_xpoly))


def fp64_peak_derived(sm_mhz=1965.0, sms=148):
    """148 SMs x 64 FP64 FMA lanes/clk x 2 flops x clock (B200 datasheet 37 TFLOP/s class)."""
    return sms * 64 * 2 * sm_mhz * 1e6 / 1e12


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = "index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap"

    def __init__(self, device_index=0):
        self.dev = device_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except (FileNotFoundError, OSError):
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax.append(float(f[2]))
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(smax), "reasons": sorted(reasons),
                "samples": len(sm)}


def load_workload(cfg, field="sinsin"):
    from paper_conf_sc_0007k13_b200 import inputs
    return inputs.make_config(cfg, field_kind=field)


def workload_desc(w, cfg):
    return {"workload": f"cfg{cfg}: {w.meta['desc']}", "n_triangles": int(len(w.T)), "n_points": int(w.n_points),
            "k": w.k, "h": w.h, "periodic": "xy", "seed": w.seed, "field": "sin(2pi x) sin(2pi y), L2-projected",
            "points": "degree-2k symmetric-rule nodes per element"}


def parity_report(g, o, tol=1e-10):
    """The parity rule of tests/test_gpu_parity.py on one sample: normwise
    max|g-o|/max|o| and pointwise |g-o|/|o| where |o| >= 1e-2 max|o|."""
    g, o = np.asarray(g, dtype=np.float64), np.asarray(o, dtype=np.float64)
    scale = max(float(np.abs(o).max()), 1e-300)
    err = np.abs(g - o)
    big = np.abs(o) >= 1e-2 * scale
    rel = err[big] / np.abs(o[big]) if big.any() else np.zeros(1)
    nw, pw = float(err.max() / scale), float(rel.max())
    return {"max_normwise": nw, "max_pointwise": pw, "p99_pointwise": float(np.quantile(rel, 0.99)),
            "n_points": int(len(o)), "tolerance": tol, "pass": bool(nw <= tol and pw <= tol and np.all(np.isfinite(g)))}


def cpu_baseline(w, idx, label, nthreads=0):
    """The oracle as it stands, on a deterministic sample `idx` of the workload's points, on
    all host cores (explicit: torchrun sets OMP_NUM_THREADS=1).  Returns the baseline record
    and the oracle's values at the sample (the bench line's parity check)."""
    import oracle
    nthreads = nthreads or oracle.omp_threads()
    P = w.points[idx]
    t0 = time.perf_counter()
    vals = oracle.oracle_eval(w.V, w.T, w.C, w.k, w.h, P, nthreads=nthreads)
    dt = time.perf_counter() - t0
    return ({"value": len(P) / dt, "unit": "points/s", "cores": nthreads, "kind": "oracle",
             "sample": f"{label} ({len(P)} points), {dt:.1f} s"}, vals)


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    w = load_workload(args.config)
    import oracle
    stride = max(1, w.n_points // args.ref_points)
    P = w.points[::stride]
    for _ in range(args.warmup):
        oracle.oracle_eval(w.V, w.T, w.C, w.k, w.h, P[:64], nthreads=oracle.omp_threads())
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.oracle_eval(w.V, w.T, w.C, w.k, w.h, P, nthreads=oracle.omp_threads())
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    val = len(P) * args.steps / tot
    line = {"metric": "filtered quadrature points/sec (FP64)", "impl": "reference", "value": val,
            "unit": "points/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * tot / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": dict(workload_desc(w, args.config), sample=f"every {stride}th point ({len(P)} points) per step"),
            "cpu_baseline": {"value": val, "unit": "points/s", "cores": oracle.omp_threads(), "kind": "oracle",
                             "sample": f"every {stride}th evaluation point ({len(P)} points) per step"},
            "e2e": {"value": val, "unit": "points/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def broadcast_workload(w, rank, device):
    """Rank 0's workload (mesh, modes, points) to every rank: the metadata by
    broadcast_object_list, the arrays by one broadcast each over the process group (NCCL over
    NVLink on a GPU box).  Returns (workload, broadcast ms of the arrays)."""
    import types

    import torch
    import torch.distributed as dist

    meta = [None]
    if rank == 0:
        meta = [{"k": w.k, "h": w.h, "seed": w.seed, "name": w.name, "meta": w.meta, "periodic": w.periodic,
                 "domain": w.domain, "shapes": {n: getattr(w, n).shape for n in ("V", "T", "C", "points")},
                 "dtypes": {n: str(getattr(w, n).dtype) for n in ("V", "T", "C", "points")}}]
    dist.broadcast_object_list(meta, src=0, device=device if device.type == "cuda" else None)
    m = meta[0]
    if device.type == "cuda":
        torch.cuda.synchronize()
    t0 = time.perf_counter()
    arrs = {}
    for n in ("V", "T", "C", "points"):
        dt = {"float64": torch.float64, "int32": torch.int32}[m["dtypes"][n]]
        if rank == 0:
            t = torch.from_numpy(np.ascontiguousarray(getattr(w, n))).to(device)
        else:
            t = torch.empty(m["shapes"][n], dtype=dt, device=device)
        dist.broadcast(t, src=0)
        arrs[n] = t
    out = {n: t.cpu().numpy() for n, t in arrs.items()}
    ms = 1e3 * (time.perf_counter() - t0)
    if rank == 0:
        return w, ms
    ns = types.SimpleNamespace(k=m["k"], h=m["h"], seed=m["seed"], name=m["name"], meta=m["meta"],
                               periodic=m["periodic"], domain=m["domain"], **out)
    ns.n_points = len(ns.points)
    return ns, ms


def run_siac(args):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_0007k13_b200 import siac

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ndev = torch.cuda.device_count()
    dev = torch.device("cuda", local % max(ndev, 1))
    torch.cuda.set_device(dev)
    backend = os.environ.get("SIAC_DIST_BACKEND", "nccl")     # gloo: functional runs with >1 rank per GPU
    if world > 1 and backend == "nccl":
        # NCCL's communicator lines (ranks, NVLink/NVLS transport) go to stderr, not the JSON stdout
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)

    def allreduce_max(vals):
        if world == 1:
            return vals
        t = torch.tensor(vals, dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return t.tolist()

    def allreduce_sum_int(vals):
        if world == 1:
            return vals
        t = torch.tensor(vals, dtype=torch.int64, device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(t)
        return [int(x) for x in t.tolist()]

    def allgather_floats(vals):
        t = torch.tensor(vals, dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
        out = torch.empty(world * len(vals), dtype=torch.float64, device=t.device)
        dist.all_gather_into_tensor(out, t)
        return out.view(world, len(vals)).tolist()

    # inputs: generated once on rank 0 and broadcast to the other ranks
    t_in = time.perf_counter()
    w = load_workload(args.config) if rank == 0 else None
    bcast_ms = None
    if world > 1:
        w, bcast_ms = broadcast_workload(w, rank, dev if backend == "nccl" else torch.device("cpu"))
    t_in = time.perf_counter() - t_in
    k = w.k
    halo_info = None
    if world > 1:
        from paper_conf_sc_0007k13_b200 import dist as sdist
        wts = sdist.work_estimate(w.V, w.T, w.points, 0.5 * (3 * k + 1) * w.h)
        part = sdist.partition(w.points, world, weights=wts)
        sub = sdist.local_problem(w.V, w.T, w.C, w.points, w.k, w.h, part, rank)
        V, T, C, P_local = sub["V"], sub["T"], sub["C"], sub["points"]
    else:
        part = None
        V, T, C, P_local = w.V, w.T, w.C, w.points
    t0 = time.perf_counter()
    ctx = siac.create(V, T, C, k, w.h, periodic=3, device=dev.index)
    create_wall_ms = 1e3 * (time.perf_counter() - t0)
    cinfo = ctx.create_info()
    ctx.set_schedule(args.schedule)
    if world > 1:
        per_rank = allgather_floats([float(len(P_local)), float(len(T)), create_wall_ms, cinfo["cross_ms"]])
        halo_info = {"points": [int(r[0]) for r in per_rank], "halo_triangles": [int(r[1]) for r in per_rank],
                     "create_ms": [round(r[2], 2) for r in per_rank],
                     "create_cross_ms": [round(r[3], 2) for r in per_rank],
                     "mesh_triangles": int(len(w.T)),
                     "input_broadcast_ms": bcast_ms}
    n_local = len(P_local)
    d_pts = torch.from_numpy(np.ascontiguousarray(P_local)).to(dev)
    d_out = torch.empty(max(n_local, 1), dtype=torch.float64, device=dev)
    stream = torch.cuda.current_stream(dev)

    # geometry counts (untimed): the algorithmic flop count of the quadrature
    ctx.set_counting(True)
    ctx.eval_async(d_pts, d_out, stream)
    st = ctx.stats()
    ctx.set_counting(False)
    cands, pairs, pieces, subtris, corners, crosses, xsub, xpoly = allreduce_sum_int(
        [st["candidates"], st["pairs"], st["pieces"], st["subtris"], st["corner_terms"], st["cross_terms"],
         st["cross_subtris"], st["cross_polys"]])
    jump = args.schedule in (0, 4, 5, 6)
    if jump:
        # JUMP: its own algorithmic flops; general-path pairs (h < triangle size only) add
        # their clip-and-integrate sub-triangles at the direct method's rate
        flops_step, unit_flops = jump_flops(k, pairs, corners, xsub, xpoly)
        flops_step += subtris * flops_per_subtri(k)
    else:
        flops_step, unit_flops = subtris * flops_per_subtri(k), (flops_per_subtri(k),)
    direct = None
    if jump and args.direct_count:
        # the direct clip-and-integrate decomposition's count (schedule TILE) for context:
        # the model flops SURVEY §8(d) defines for the same integral
        ctx.set_schedule(2)
        ctx.set_counting(True)
        ctx.eval_async(d_pts, d_out, stream)
        sd = ctx.stats()
        ctx.set_counting(False)
        ctx.set_schedule(args.schedule)
        d_pieces, d_sub = allreduce_sum_int([sd["pieces"], sd["subtris"]])
        direct = {"pieces": d_pieces, "subtris": d_sub, "model_flops_per_step": d_sub * flops_per_subtri(k)}

    # per-step gather of the values (NCCL all_gather_into_tensor of padded slices)
    if world > 1:
        nmax = part["max_count"]
        gdev = dev if backend == "nccl" else torch.device("cpu")
        send = torch.zeros(nmax, dtype=torch.float64, device=gdev)
        gathered = torch.empty(world * nmax, dtype=torch.float64, device=gdev)

    def gather(vals_dev):
        if world > 1:
            send[:n_local].copy_(vals_dev[:n_local])
            dist.all_gather_into_tensor(gathered, send)

    # L2: flush between timed steps unless this rank's inputs alone exceed the 126 MB L2
    in_bytes = n_local * 16 + len(T) * cinfo["bytes_per_triangle"]
    flush = in_bytes < 2 * 126e6
    scrub = torch.empty(int(256e6) // 4, dtype=torch.float32, device=dev) if flush else None

    for _ in range(args.warmup):
        ctx.eval_async(d_pts, d_out, stream)
        gather(d_out)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ctx.timing()                       # discard
    ctx.set_timing(True)
    clocks = ClockSampler(dev.index)
    clocks.start()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    for i in range(args.steps):
        if flush:
            scrub.fill_(float(i))      # write 256 MB > L2 between timed steps (outside the events)
        ev[i][0].record(stream)
        ctx.eval_async(d_pts, d_out, stream)
        gather(d_out)
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    ms_total = sum(a.elapsed_time(b) for a, b in ev)
    kern_ms, kern_n = ctx.timing()
    ctx.set_timing(False)
    ms_total, kern_ms = allreduce_max([ms_total, kern_ms])
    ms_step = ms_total / args.steps
    value = w.n_points / (ms_step * 1e-3)

    # the values of the last timed step, for the parity check (N > 1: assembled from the gather)
    vals_local = d_out[:n_local].cpu().numpy()
    vals_full = None
    if world > 1 and rank == 0:
        vals_full = sdist.assemble(gathered.cpu().numpy(), part, w.n_points)

    # end-to-end through the public host-buffer API (siac_eval): every step copies this rank's
    # points from pinned host memory, evaluates, copies the values back, and (N > 1) gathers
    # all ranks' values so every rank holds the full result
    h_pts = torch.from_numpy(np.ascontiguousarray(P_local)).pin_memory()
    h_out = torch.empty(max(n_local, 1), dtype=torch.float64).pin_memory()
    hp, ho = h_pts.numpy().reshape(-1, 2), h_out.numpy()
    ctx.eval_into(hp, ho)
    if world > 1:
        gather(h_out.to(gathered.device))
        torch.cuda.synchronize()
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(args.e2e_steps):
        ctx.eval_into(hp, ho)
        if world > 1:
            gather(h_out.to(gathered.device, non_blocking=False))
            full = gathered.cpu()
    e2e_s = allreduce_max([time.perf_counter() - t0])[0]
    e2e_val = w.n_points / (e2e_s / args.e2e_steps) if args.e2e_steps > 0 else None
    ctx.destroy()

    # one-shot use (the paper's: one evaluation at the end of a run):
    # siac_create from host arrays + siac_eval (host buffers) + siac_destroy, per rank, then the
    # gather; max over ranks
    oneshot = None
    if args.oneshot:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        c1 = siac.create(V, T, C, k, w.h, periodic=3, device=dev.index)
        c1.set_schedule(args.schedule)
        c1.eval_into(hp, ho)
        c1.destroy()
        if world > 1:
            gather(h_out.to(gathered.device, non_blocking=False))
            full = gathered.cpu()
        os_s = allreduce_max([time.perf_counter() - t0])[0]
        oneshot = {"ms": 1e3 * os_s, "value": w.n_points / os_s, "unit": "points/s",
                   "note": "siac_create (host arrays) + siac_eval (host buffers) + siac_destroy"
                           + (" + all_gather, max over ranks" if world > 1 else "")}

    peak_meas = siac.probe_fp64(dev.index)
    line = None
    if rank == 0:
        kern_avg_s = (kern_ms / max(kern_n, 1)) * 1e-3
        # whole-job algorithmic flops per launch-set / slowest rank's kernel time / ranks
        achieved = flops_step / world / kern_avg_s / 1e12 if kern_avg_s > 0 else None
        peak = fp64_peak_derived()
        # DRAM traffic per launch from the committed ncu --set full capture of this kernel at
        # the bench's own cfg-5 launch (profiles/*_ncu_traffic_cfg5.json), scaled by points
        traffic, ncu_rec = None, None
        for tp in ("r02g_ncu_traffic_cfg5.json", "r02b_ncu_traffic_cfg5.json", "r02_ncu_traffic_cfg5.json", "r01_ncu_traffic_jumpx.json"):
            tpath = os.path.join(ROOT, "profiles", tp)
            if args.schedule in (0, 5) and os.path.exists(tpath):
                ncu_rec = json.load(open(tpath))
                ncu_rec["file"] = "profiles/" + tp
                traffic = ncu_rec["bytes_per_point"] * n_local
                break
        alg_bytes = 28 * n_local + len(T) * cinfo["bytes_per_triangle"]
        cfgd = workload_desc(w, args.config)
        cfgd.update({"parallelism": f"spatial point tiles x{world} + halo, NCCL all_gather" if world > 1
                     else "single GPU",
                     "l2": ("L2 flushed (256 MB write) between timed steps" if flush else
                            "inputs larger than L2 (points %.0f MB + triangle records %.0f MB > 126 MB)"
                            % (n_local * 16 / 1e6, len(T) * cinfo["bytes_per_triangle"] / 1e6)),
                     "counts": {"candidates": cands, "pairs": pairs, "pieces": pieces, "subtris": subtris,
                                "corner_terms": corners, "cross_terms": crosses, "cross_subtris": xsub,
                                "cross_polys": xpoly},
                     "flops_per_unit": dict(zip(["pair", "corner", "cross_subtri", "cross_poly"] if jump
                                                else ["subtri"], unit_flops))})
        line = {"metric": "filtered quadrature points/sec (FP64)", "value": value, "unit": "points/s",
                "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic", "config": cfgd,
                "roofline": {"bound": "alu", "kernel": "k_eval", "achieved": achieved, "peak": peak,
                             "unit": "TFLOP/s", "frac": (achieved / peak) if achieved else None, "traffic": traffic,
                             "traffic_note": ("dram read+write bytes per launch from the committed ncu --set full "
                                              "capture (%s), scaled by this launch's points" % (ncu_rec["file"] if ncu_rec else "none")),
                             # compulsory bytes of one launch: points (16 B) + permutation (4 B) + values (8 B)
                             # per point, and every resident triangle record read at least once
                             "algorithmic_bytes": alg_bytes,
                             "traffic_over_algorithmic": (traffic / alg_bytes) if traffic else None,
                             "peak_note": "derived: 148 SM x 64 FP64 FMA/clk x 2 x 1965 MHz (DESIGN.md §8.1)",
                             "measured_dfma_peak": peak_meas,
                             "frac_of_measured": (achieved / peak_meas) if achieved else None,
                             "kernel_share_of_step": (kern_ms / kern_n) / ms_step if kern_n else None,
                             "algorithmic_flops_per_step": flops_step,
                             "flop_model": ("headline: the JUMP decomposition's own operation count (DESIGN.md "
                                            "§8.2); see direct_method for SURVEY §8(d)'s per-quadrature-point model "
                                            "and ncu_executed for the executed FP64 instructions" if jump else
                                            "direct SH + fan + quadrature (SURVEY §8(d))")},
                "create": {"wall_ms": create_wall_ms, **{k_: cinfo[k_] for k_ in
                           ("host_ms", "h2d_ms", "index_ms", "jump_ms", "cross_ms", "device_bytes",
                            "bytes_per_triangle")},
                           "cross_share_of_eval_step": cinfo["cross_ms"] / ms_step,
                           "note": "siac_create once per mesh, excluded from value (SURVEY §8(d)); rank 0's"},
                "e2e": {"value": e2e_val, "unit": "points/s", "h2d_bytes_per_step": int(w.n_points * 16),
                        "d2h_bytes_per_step": int(w.n_points * 8)},
                "oneshot": oneshot,
                "schedule": ["default(jump-x)", "point", "tile", "ws", "jump", "jump-x", "elem"][args.schedule],
                "gpu_launches": 2 * args.steps,
                "gpu_launches_note": "per step and rank: k_point_keys + k_eval (ours) + CUB radix-sort kernels",
                "clocks": clk}
        if ncu_rec is not None and ncu_rec.get("fp64_executed_tflops_equiv") is not None:
            line["roofline"]["ncu_executed"] = {
                "fp64_pipe_pct": ncu_rec.get("fp64_pipe_pct"),
                "executed_frac": ncu_rec.get("fp64_executed_frac"),
                "note": "(2 DFMA + DADD + DMUL) thread instructions / kernel time / derived peak, ncu capture"}
        if halo_info is not None:
            line["multi_gpu"] = halo_info
        if direct is not None:
            dm = direct["model_flops_per_step"]
            direct["model_tflops_equivalent"] = dm / world / kern_avg_s / 1e12 if kern_avg_s > 0 else None
            direct["model_frac"] = direct["model_tflops_equivalent"] / peak if kern_avg_s > 0 else None
            direct["note"] = ("SURVEY §8(d) model flops of the direct decomposition of the same integral / this "
                              "kernel's time: the work the jump decomposition avoids, not executed flops")
            line["direct_method"] = direct
    if rank == 0 and not args.no_cpu_baseline:
        if world == 1:
            # the oracle timed on a stride sample, and the GPU's values at the same points
            stride = max(1, w.n_points // args.ref_points)
            idx = np.arange(0, w.n_points, stride)
            cb, ovals = cpu_baseline(w, idx, f"every {stride}th evaluation point")
            line["cpu_baseline"] = cb
            line["parity"] = dict(parity_report(vals_local[idx], ovals), sample=cb["sample"])
        else:
            # N > 1: the assembled (gathered) values against the oracle on points next to the
            # partition cuts (their values depend on the halos) plus a stride sample
            hw = 0.5 * (3 * k + 1) * w.h
            near = sdist.near_cut_points(w.points, part, hw)
            rng = np.random.default_rng(77)
            pick = np.sort(rng.choice(near, size=min(len(near), args.ref_points // 4), replace=False))
            idx = np.unique(np.concatenate([pick, np.arange(0, w.n_points, max(1, 4 * w.n_points // args.ref_points))]))
            _, ovals = cpu_baseline(w, idx, "near-cut + stride")
            line["parity"] = dict(parity_report(vals_full[idx], ovals),
                                  sample=f"{len(pick)} points within W/2 of the {world}-way partition cuts + a stride "
                                         f"sample, gathered values")
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--impl", default="siac", choices=["siac", "reference"])
    ap.add_argument("--ref-points", type=int, default=4000, help="oracle sample size (points)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--schedule", type=int, default=0,
                    help="0 = default (jump-x), 1 = thread-per-point, 2 = warp-per-tile, 3 = warp-specialized, "
                         "4 = jump, 5 = jump with closed-form cross terms, 6 = per-element (scatter)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-oneshot", dest="oneshot", action="store_false",
                    help="skip the one-shot create + eval + destroy timing")
    ap.add_argument("--no-direct-count", dest="direct_count", action="store_false",
                    help="skip the (untimed) direct-decomposition count run")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    return run_siac(args)


if __name__ == "__main__":
    sys.exit(main())
