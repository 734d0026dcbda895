#!/usr/bin/env python3
"""Build an experimental variant of the library with extra -D flags:
python tools/build_variant.py NAME -DFOO=1 ...  -> paper_conf_sc_0007k13_b200/libsiac_b200.NAME.so"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sc_0007k13_b200")
name, defs = sys.argv[1], sys.argv[2:]
obj = os.path.join(PKG, "csrc", f"siac_math.{name}.o")
subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-c", "-o", obj, os.path.join(PKG, "csrc", "siac_math.cpp")])
cmd = ["nvcc", "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-Xcompiler", "-fPIC",
       "-shared", "-Xptxas", "-v"] + defs + ["-o", os.path.join(PKG, f"libsiac_b200.{name}.so"),
                                             os.path.join(PKG, "csrc", "siac.cu"), obj]
out = subprocess.run(cmd, capture_output=True, text=True)
if out.returncode:
    print(out.stderr)
    sys.exit(1)
lines = out.stderr.splitlines()
for i, l in enumerate(lines):
    if "Function properties for" in l and "k_eval_tileILi3ELb0" in l:
        print(name, lines[i + 1].strip(), "|", lines[i + 2].strip())
