"""Per-instruction executed counts of an ncu capture, grouped by execution
frequency band and by opcode (reads `ncu --page source --print-source sass`).
usage: python tools/sass_hot.py report.ncu-rep [per_unit_count] [--dump LO HI]"""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr = rows[1]
ie, src = hdr.index("Instructions Executed"), hdr.index("Source")
seq = []
for r in rows[2:]:
    try:
        seq.append((int(r[ie]), r[src].strip()))
    except (ValueError, IndexError):
        pass
tot = sum(n for n, _ in seq)
print("total warp instructions", tot)
ops = collections.Counter()
for n, s in seq:
    t = s.split()
    if not t:
        continue
    op = t[1] if t[0].startswith("@") and len(t) > 1 else t[0]
    ops[op.split(".")[0]] += n
for o, n in ops.most_common(20):
    print(f"  {o:12s} {n:12d} {100 * n / tot:5.1f}%")
if "--dump" in sys.argv:
    i = sys.argv.index("--dump")
    lo, hi = int(sys.argv[i + 1]), int(sys.argv[i + 2])
    for n, s in seq:
        if lo <= n < hi:
            print(n, s[:100])
else:
    bands = collections.Counter()
    for n, s in seq:
        bands[10 ** len(str(n)) if n else 0] += n
    for b in sorted(bands):
        print(f"  count < {b:>12d}: {bands[b]:12d} ({100 * bands[b] / tot:4.1f}%)")
