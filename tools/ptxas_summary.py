#!/usr/bin/env python3
"""Registers / spills / stack per kernel entry from an `nvcc -Xptxas -v` log.
    python tools/ptxas_summary.py build/libfpx.ptxas.txt [filter]"""
import re
import sys

txt = open(sys.argv[1]).read().splitlines()
flt = sys.argv[2] if len(sys.argv) > 2 else ""
cur = None
info = {}
for line in txt:
    m = re.search(r"Compiling entry function '([^']+)'", line)
    if m:
        cur = m.group(1)
        info[cur] = {}
        continue
    if cur is None:
        continue
    m = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m and "stack" not in info[cur]:
        info[cur]["stack"], info[cur]["spill_st"], info[cur]["spill_ld"] = map(int, m.groups())
    m = re.search(r"Used (\d+) registers", line)
    if m and "regs" not in info[cur]:
        info[cur]["regs"] = int(m.group(1))
for k, v in info.items():
    if flt in k:
        name = re.sub(r"_ZN3fpx\d+_GLOBAL__N__\w+?_\d+_fpx_\w+?_cu_\w+?(\d+k_)", r"\1", k)
        print(f"{name[:110]:110s} regs {v.get('regs')} stack {v.get('stack')} spill {v.get('spill_st')}/{v.get('spill_ld')}")
