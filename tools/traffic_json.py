"""Rewrite profiles/traffic.json from the per-config DRAM traffic captures of one
gpurun session (tools/gpu_check.sh with NCU_TRAFFIC=1).

    python tools/traffic_json.py gpurun_out/<tag> [config ...]

Each gpurun_out/<tag>/traffic_<config>.csv holds one ncu launch (the 5th, after
4 warm-up steps) with dram__bytes_read.sum, dram__bytes_write.sum and
gpu__time_duration.sum; bench.py reports read + write as roofline.traffic.
Configs not captured in this session keep their previous entry."""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src = sys.argv[1]
out = os.path.join(ROOT, "profiles", "traffic.json")
tj = json.load(open(out)) if os.path.exists(out) else {}
cfgs = sys.argv[2:] or sorted(f[len("traffic_"):-4] for f in os.listdir(src) if f.startswith("traffic_") and f.endswith(".csv"))
for c in cfgs:
    rows = list(csv.reader(open(os.path.join(src, f"traffic_{c}.csv"))))
    hdr = next(r for r in rows if "Metric Name" in r)
    iname, ival, ikern = hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("Kernel Name")
    vals, kern = {}, None
    for r in rows[rows.index(hdr) + 1:]:
        if len(r) > ival:
            vals[r[iname]] = float(r[ival].replace(",", ""))
            kern = r[ikern]
    rd, wr = int(vals["dram__bytes_read.sum"]), int(vals["dram__bytes_write.sum"])
    ent = {"kernel": kern, "dram_bytes_read": rd, "dram_bytes_write": wr, "dram_bytes_per_launch": rd + wr,
           "ncu_duration_ns": int(vals["gpu__time_duration.sum"]), "source": os.path.relpath(src, ROOT)}
    if "algorithmic_bytes" in tj.get(c, {}):
        ent["algorithmic_bytes"] = tj[c]["algorithmic_bytes"]
    tj[c] = ent
tj["about"] = ("DRAM bytes (read + write) per launch of the dominant kernel at the full bench configuration; "
               "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none, "
               "5th launch (after 4 warm-up steps); written by tools/traffic_json.py from gpurun_out/<tag>/traffic_*.csv "
               "(`source`); the csv copies are in profiles/r1/.")
json.dump(tj, open(out, "w"), indent=1)
print(json.dumps(tj, indent=1))
