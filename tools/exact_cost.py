"""Cost of the record scan's exact path per storm record, by mode.

    python tools/exact_cost.py [n_records] [n_storms]

A FLOW-recipe trace (FP32 / FP64 records with 1..3 sources) is scanned clean,
then with whole-warp storms planted (fpxgen.plan_injections, storm_frac = 1);
(time with storms - clean time) x warps / storm records = the exact path's
cost per storm record for one warp, in DEST, FLOW and FLOW_DETAIL modes."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import fpxgen  # noqa: E402
from paper_conf_hpdc_lilfslg23_b200 import fpx  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 4_000_000
n_storms = int(sys.argv[2]) if len(sys.argv) > 2 else 3_000
WARPS = 148 * 20


def timed(h, hdr, arena, planes, mode, reps=20):
    s = torch.cuda.current_stream()
    ts = []
    for i in range(reps + 3):
        h.reset(stream=s)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        h.scan_records(hdr, arena, mode=mode, arena_planes=planes, stream=s)
        b.record(s)
        torch.cuda.synchronize()
        if i >= 3:
            ts.append(a.elapsed_time(b))
    return float(np.median(ts))


p = fpxgen.Params(seed=77, n_records=n, n_sites=1_000, recipe=fpxgen.RECIPE_FLOW, p_fp64=0.3)
hdr, arena, planes = fpxgen.generate_device(p)
clean = {}
with fpx.Handle(0) as h:
    for mode in (0, 1, 2):
        clean[mode] = timed(h, hdr, arena, planes, mode)
inj, w = fpxgen.plan_injections(p, n_storms, storm_frac=1.0, flow=True)
fpxgen.apply_device(w, hdr, arena)
storm_recs = len(np.unique(inj["record"]))
with fpx.Handle(0) as h:
    for mode, name in ((0, "DEST"), (1, "FLOW"), (2, "FLOW_DETAIL")):
        t = timed(h, hdr, arena, planes, mode)
        extra = (t - clean[mode]) * 1e3  # us
        print(f"{name:12s} clean {clean[mode] * 1e3:8.1f} us  storms {t * 1e3:8.1f} us  "
              f"storm records {storm_recs}  exact cost {extra * WARPS / max(storm_recs, 1):6.2f} us per record per warp",
              flush=True)
