#!/usr/bin/env python3
"""Registers / spills per kernel instantiation from an nvcc -Xptxas -v log (demangled)."""
import re
import subprocess
import sys

txt = open(sys.argv[1]).read()
pat = sys.argv[2] if len(sys.argv) > 2 else ""
for b in re.split(r"ptxas info    : Compiling entry function '", txt)[1:]:
    name = b.split("'")[0]
    dem = subprocess.run(["cu++filt", name], capture_output=True, text=True).stdout.strip()
    dem = re.sub(r"lt::<unnamed>::|\(int\)|void ", "", dem)
    if pat not in dem:
        continue
    r = re.search(r"Used (\d+) registers", b)
    st = re.search(r"(\d+) bytes spill stores", b)
    ld = re.search(r"(\d+) bytes spill loads", b)
    print(f"{dem.split('(')[0]:55s} regs {r.group(1) if r else '?':>4} spill st {st.group(1) if st else '?':>4} ld {ld.group(1) if ld else '?':>4}")
