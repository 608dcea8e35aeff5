#!/usr/bin/env python3
"""Table of the storm captures of tools/storm_ncu.sh (one ncu launch per
config: duration, warp instructions, L2 atomic / reduction requests, shared
atomics, L2 atomic-unit activity) plus the bench line of each config.
    python tools/storm_summary.py gpurun_out/<tag>/storm [gpurun_out/<tag>/storm_noagg]"""
import csv
import json
import os
import sys

KEYS = [("gpu__time_duration.sum", "ncu_us", 1e-3), ("smsp__inst_executed.sum", "warp_inst_M", 1e-6),
        ("lts__t_requests_srcunit_tex_op_atom.sum", "L2_atom_req", 1), ("lts__t_requests_srcunit_tex_op_red.sum", "L2_red_req", 1),
        ("smsp__sass_inst_executed_op_global_atom.sum", "g_atom_inst", 1),
        ("smsp__sass_inst_executed_op_global_red.sum", "g_red_inst", 1),
        ("smsp__sass_inst_executed_op_shared_atom.sum", "s_atom_inst", 1),
        ("lts__d_atomic_input_cycles_active.avg.pct_of_peak_sustained_elapsed", "L2_atom_unit_%", 1),
        ("smsp__issue_active.avg.pct_of_peak_sustained_elapsed", "issue_%", 1)]
for d in sys.argv[1:]:
    tag = "no warp aggregation (FPX_OPT_NO_WARP_AGG)" if "noagg" in d else "default (warp + CTA aggregation)"
    print(f"# {tag}: {d}")
    for f in sorted(os.listdir(d)):
        if not (f.startswith("ncu_") and f.endswith(".csv")):
            continue
        cfg = f[4:-4]
        rows = [r for r in csv.reader(open(os.path.join(d, f))) if len(r) > 5]
        h = rows[0]
        v = {r[h.index("Metric Name")]: float(r[h.index("Metric Value")].replace(",", "")) for r in rows[1:]}
        b = {}
        bp = os.path.join(d, f"bench_{cfg}.json")
        if os.path.exists(bp):
            try:
                b = json.loads(open(bp).read())
            except ValueError:
                pass
        line = f"{cfg:4s}"
        if b:
            line += f" bench {b['roofline']['kernel_ms']:.4f} ms {b['roofline']['achieved']:.0f} GB/s (frac {b['roofline']['frac']:.3f})"
        for k, name, sc in KEYS:
            if k in v:
                x = v[k] * sc
                line += f" {name} {x:.4g}"
        print(line)
