#!/usr/bin/env python3
"""Summarise an ncu report: key raw metrics + SASS opcode stall histogram + top stall PCs.
usage: python tools/ncu_summary.py report.ncu-rep [top]"""
import csv
import io
import subprocess
import sys
from collections import Counter

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = r[0], r[1], r[2]
KEYS = ["gpu__time_duration.sum", "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fp64.avg.pct", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "smsp__inst_executed.sum", "smsp__issue_active.avg.pct", "sass__inst_executed_local", "dram__bytes_read.sum",
        "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
        "launch__grid_size", "launch__block_size", "sm__throughput.avg.pct", "launch__shared_mem_per_block"]
print("== raw metrics")
for i, h in enumerate(hdr):
    if any(h.startswith(k) for k in KEYS) and not h.endswith(("per_second", ".max", ".min")):
        print(f"  {h} [{units[i]}] = {vals[i]}")
print("== stall reasons (warps per issue-active cycle)")
st = []
for i, h in enumerate(hdr):
    if h.startswith("smsp__average_warps_issue_stalled") and h.endswith("_per_issue_active.ratio"):
        try:
            st.append((float(vals[i]), h.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", "")))
        except ValueError:
            pass
for v, n in sorted(st, reverse=True)[:10]:
    print(f"  {n:28s} {v:.3f}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
h = rows[1]
si, wi, ei = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
cat, cnt, data, tot = Counter(), Counter(), [], 0
for row in rows[2:]:
    if len(row) <= wi:
        continue
    s = row[si].strip()
    w = int(row[wi] or 0)
    e = int(row[ei] or 0)
    parts = s.split()
    op = parts[1] if parts and parts[0].startswith("@") and len(parts) > 1 else (parts[0] if parts else "")
    base = op.split(".")[0]
    cat[base] += w
    cnt[base] += e
    tot += w
    data.append((w, row[0], s))
print(f"== stall samples by opcode (total {tot})")
for k, v in cat.most_common(top):
    print(f"  {k:10s} {100 * v / max(tot, 1):5.1f}%  exec {cnt[k]}")
data.sort(reverse=True)
print("== top PCs")
for w, a, s in data[:top]:
    print(f"  {w:8d} {a[-6:]} {s[:90]}")

# ---- per CUDA source line (needs -lineinfo): stall samples aggregated by file:line
cs = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                    capture_output=True, text=True).stdout
lines, fname = [], "?"
hdr = None
for row in csv.reader(io.StringIO(cs)):
    if not row:
        continue
    if row[0] == "File Path":
        fname = row[1].split("/")[-1]
        continue
    if row[0] == "Line No":
        hdr = row
        continue
    if hdr is None or row[0] == "Function Name" or not row[0].isdigit():
        continue
    try:
        w = int(row[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
        e = int(row[hdr.index("Instructions Executed")] or 0)
    except (ValueError, IndexError):
        continue
    lines.append((w, e, f"{fname}:{row[0]}", row[1][:70]))
lines.sort(reverse=True)
tot = sum(x[0] for x in lines)
print(f"== top source lines by stall samples (total {tot})")
for w, e, loc, src in lines[:top]:
    print(f"  {100 * w / max(tot, 1):5.1f}% exec {e:>12d}  {loc:22s} {src}")
