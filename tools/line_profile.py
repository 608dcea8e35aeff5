#!/usr/bin/env python3
"""Warp instructions executed per CUDA source line, for one kernel of an ncu
capture (`ncu --set full --import-source on`): joins ncu's per-SASS-instruction
counts with `nvdisasm -gi` line info of the same library build.

    python tools/line_profile.py report.ncu-rep lib.so [kernel-substring] [--top N] [--outer] [--col NAME]

--outer aggregates by the outermost source line (the kernel body line an
inlined call sits on) instead of the innermost one; --col aggregates another per-instruction column
of the source page (e.g. "Warp Stall Sampling (All Samples)", "stall_long_sb")."""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

rep, lib = sys.argv[1], sys.argv[2]
ksub = sys.argv[3] if len(sys.argv) > 3 and not sys.argv[3].startswith("--") else ""
top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 40
outer = "--outer" in sys.argv
col = sys.argv[sys.argv.index("--col") + 1] if "--col" in sys.argv else "Instructions Executed"

txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
kname = rows[0][1] if rows and len(rows[0]) > 1 else ""
hdr = rows[1]
ie, src = hdr.index(col), hdr.index("Source")
counts = []
for r in rows[2:]:
    try:
        counts.append((int(r[ie]), r[src].strip()))
    except (ValueError, IndexError):
        pass

tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=tmp, capture_output=True)
cubins = [f for f in os.listdir(tmp) if f.endswith(".cubin") and "-" not in f]
best = None
for cb in cubins:
    dis = subprocess.run(["nvdisasm", "-gi", os.path.join(tmp, cb)], capture_output=True, text=True).stdout
    # functions: ".text.<mangled>:" then instructions "/*0040*/ OP ..."
    funcs = re.split(r"\n\.text\.(\S+):\n", dis)
    for i in range(1, len(funcs), 2):
        name, body = funcs[i], funcs[i + 1]
        if ksub and ksub not in name:
            continue
        cur_in, cur_out = None, None
        fresh = True  # the first //## line after an instruction is the innermost; later ones walk outwards
        ins = []
        for line in body.splitlines():
            m = re.match(r'\s*//## File "([^"]+)", line (\d+)(?: inlined at "([^"]+)", line (\d+))?', line)
            if m:
                here = (os.path.basename(m.group(1)), int(m.group(2)))
                if fresh:
                    cur_in = here
                    fresh = False
                cur_out = (os.path.basename(m.group(3)), int(m.group(4))) if m.group(3) else here
                continue
            m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
            if m:
                ins.append((m.group(2).strip(), cur_in, cur_out))
                fresh = True
        if len(ins) >= len(counts) * 0.9 and len(ins) <= len(counts) * 1.1:
            best = ins
            break
    if best:
        break
if not best:
    sys.exit("no function in the library matches the capture's instruction count (same build?)")

agg = collections.Counter()
tot = sum(n for n, _ in counts)
for (n, s), (op, li, lo) in zip(counts, best):
    key = lo if outer else li
    agg[key] += n
print(f"kernel {kname[:100]}  total {col} {tot}")
for k, n in agg.most_common(top):
    print(f"  {n:12d} {100 * n / tot:5.1f}%  {k}")
