#!/usr/bin/env python3
"""Per-source-line SASS opcode counts of one kernel: joins an ncu source page (sass view, with
'Instructions Executed') to a local nvdisasm --print-line-info listing of the same binary.
usage: python tools/sass_lines.py ncu_sass.csv local.sass FUNC_MANGLED NORM [file:lo-hi ...]"""
import collections
import csv
import re
import sys

sass_csv, listing, fn, norm = sys.argv[1], sys.argv[2], sys.argv[3], float(sys.argv[4])
lines = open(listing).read().split('\n')
start = [i for i, l in enumerate(lines) if l.startswith('.text.' + fn + ':')][0]
cur, instrs = None, []
for l in lines[start + 1:]:
    if l.startswith('.text.') or l.startswith('//----'):
        break
    m = re.match(r'\s*//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (m.group(1).split('/')[-1], int(m.group(2)))
        continue
    m = re.match(r'\s*/\*([0-9a-f]{4,})\*/\s+(.*?);', l)
    if m:
        instrs.append((cur, m.group(2).strip()))
rows = list(csv.reader(open(sass_csv)))
hdr = rows[1]
ie = hdr.index("Instructions Executed")
ex = [int(r[ie]) for r in rows[2:] if len(r) > ie and r[ie].isdigit()]
assert len(ex) == len(instrs), (len(ex), len(instrs))
per = collections.defaultdict(collections.Counter)
for (loc, ins), n in zip(instrs, ex):
    per[loc][re.sub(r'^@!?U?P\w+\s+', '', ins).split()[0]] += n
tot = sum(ex)
print(f"total {tot / norm:.1f} per unit")
for loc in sorted(per, key=lambda x: (x or ('', 0))):
    c = per[loc]
    s = sum(c.values())
    if s / norm < 0.3:
        continue
    top = " ".join(f"{k}:{v / norm:.1f}" for k, v in c.most_common(6))
    print(f"{s / norm:6.1f} {loc[0] if loc else '?'}:{loc[1] if loc else 0}  {top}")
