#!/usr/bin/env python3
"""Build an experimental variant of the library with extra -D flags:
python tools/build_variant.py NAME -DFOO=1 ...  -> paper_conf_sc_0007k13_b200/libsiac_b200.NAME.so
(load it with SIAC_LIB_VARIANT=NAME)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_0007k13_b200 import siac  # noqa: E402

name, defs = sys.argv[1], sys.argv[2:]
out = os.path.join(os.path.dirname(siac.LIB_PATH), f"libsiac_b200.{name}.so")
print(siac.build(extra_flags=defs, out_path=out))
