#!/usr/bin/env python3
"""DRAM traffic and executed FP64 work of one captured k_eval launch (ncu --set full plus the
DFMA/DADD/DMUL thread-instruction metrics), written as the JSON bench.py reads for its
roofline.traffic / roofline.ncu_executed fields.

usage: python tools/ncu_traffic.py report.ncu-rep N_POINTS CAPTURE_DESCRIPTION out.json
"""
import csv
import io
import json
import subprocess
import sys


def main():
    rep, npts, desc, out = sys.argv[1], int(sys.argv[2]), sys.argv[3], sys.argv[4]
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    hdr, units, vals = r[0], r[1], r[2]

    def get(name):
        i = hdr.index(name)
        v = float(vals[i].replace(",", ""))
        u = units[i]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ms": 1e-3, "us": 1e-6, "usecond": 1e-6,
                 "msecond": 1e-3, "nsecond": 1e-9, "ns": 1e-9, "s": 1.0, "second": 1.0, "inst": 1, "": 1,
                 "%": 1, "Kinst": 1e3, "Minst": 1e6, "Ginst": 1e9}.get(u, 1)
        return v * scale

    t = get("gpu__time_duration.sum")
    rd, wr = get("dram__bytes_read.sum"), get("dram__bytes_write.sum")
    fma = get("smsp__sass_thread_inst_executed_op_dfma_pred_on.sum")
    add = get("smsp__sass_thread_inst_executed_op_dadd_pred_on.sum")
    mul = get("smsp__sass_thread_inst_executed_op_dmul_pred_on.sum")
    flops = 2 * fma + add + mul
    peak = 148 * 64 * 2 * 1965e6
    kname = r[2][hdr.index("Kernel Name")] if "Kernel Name" in hdr else "k_eval"
    rec = {"kernel": kname, "capture": desc, "points": npts, "kernel_ms": 1e3 * t,
           "dram_read_bytes": rd, "dram_write_bytes": wr, "bytes_per_point": (rd + wr) / npts,
           "fp64_thread_inst": {"dfma": fma, "dadd": add, "dmul": mul},
           "fp64_executed_tflops_equiv": flops / t / 1e12, "fp64_executed_frac": flops / t / peak,
           "fp64_pipe_pct": get("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"),
           "issue_active_pct": get("smsp__issue_active.avg.pct_of_peak_sustained_active"),
           "warps_active_pct": get("sm__warps_active.avg.pct_of_peak_sustained_active"),
           "registers_per_thread": get("launch__registers_per_thread"),
           "l2_hit_pct": get("lts__t_sector_hit_rate.pct"),
           "note": "ncu serialises and replays the launch (clock-control none): its absolute time is not a "
                   "bench number; the per-launch bytes and instruction counts are"}
    print(json.dumps(rec, indent=1))
    with open(out, "w") as f:
        json.dump(rec, f, indent=1)


if __name__ == "__main__":
    main()
