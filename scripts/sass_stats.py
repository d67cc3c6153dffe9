#!/usr/bin/env python
"""Opcode histogram of a specialization's SASS (CPU: real NVRTC, fake load/launch).
  python scripts/sass_stats.py micro_column [all|none]"""
import collections
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import test_nvrtc_specialize as T  # noqa: E402

entry = sys.argv[1]
mode = sys.argv[2] if len(sys.argv) > 2 else "all"
d = tempfile.mkdtemp()
cubin, _ = T.compile_case(entry, mode, d)
s = T.sass(cubin, d)
ops = collections.Counter()
for line in s.splitlines():
    m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_.]+)", line)
    if m:
        ops[m.group(2).split(".")[0]] += 1
print(sum(ops.values()), "static instructions")
for op, n in ops.most_common(40):
    print(f"{op:12s} {n}")
