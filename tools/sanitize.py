"""Small scans of every kernel family for compute-sanitizer (memcheck,
racecheck, synccheck): DEST / FLOW / FLOW_DETAIL record scans (TMA ring and
LDG), the record scan's dynamic tail, storm traces through the sparse and the
storm DEST kernels (exact path, CTA table, table atomics), tensor scans with ragged
heads / tails, fetch / FETCH_NEW / reset / merge paths."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import fpxgen  # noqa: E402
from paper_conf_hpdc_lilfslg23_b200 import fpx  # noqa: E402

dev = torch.device("cuda", 0)
for recipe, mode in ((fpxgen.RECIPE_MIX, 0), (fpxgen.RECIPE_FLOW, 1), (fpxgen.RECIPE_FLOW, 2), (fpxgen.RECIPE_PACKED, 0)):
    p = fpxgen.Params(seed=recipe, n_records=20_011, n_sites=300, recipe=recipe)
    hdr, arena, planes = fpxgen.generate_device(p)
    _, w = fpxgen.plan_injections(p, 200, flow=recipe == fpxgen.RECIPE_FLOW)
    fpxgen.apply_device(w, hdr, arena)
    for flags in (0, fpx.OPT_SCAN_LDG):
        with fpx.Handle(0, flags=flags) as h:
            h.scan_records(hdr, arena, mode=mode, arena_planes=planes)
            e = h.fetch()
            n = h.fetch_new()
            k, c, f = h.fetch_device()
            u = h.unique_device(torch.cat([k, k]))
            c2, f2 = h.lookup_device(u)
            h.reset()
            h.merge_device(k, c, f)
            assert len(h.fetch()) == len(e) == len(n)
# the record scan's dynamic tail (>= 148 x 20 x 512 records): chunks claimed by
# atomics, counters re-armed by the last warp; two launches back to back
p = fpxgen.Params(seed=11, n_records=1_520_011, n_sites=300, recipe=fpxgen.RECIPE_MIX, p_fp64=0.5)
hdr, arena, planes = fpxgen.generate_device(p)
_, w = fpxgen.plan_injections(p, 500)
fpxgen.apply_device(w, hdr, arena)
with fpx.Handle(0) as h:
    for _ in range(2):
        h.scan_records(hdr, arena, arena_planes=planes)
    h.fetch()
del hdr, arena
p = fpxgen.Params(seed=9, n_records=5000, n_sites=20, recipe=fpxgen.RECIPE_STRESS, dense_nan=1.0)
hdr, arena, planes = fpxgen.generate_device(p)
for flags in (0, fpx.OPT_STORM):  # the small-trace ring: sparse and storm DEST kernels
    with fpx.Handle(0, table_log2_slots=5, flags=flags) as h:
        h.scan_records(hdr, arena, arena_planes=planes)
        h.fetch()
# storms: the storm DEST kernel (CTA pre-aggregation table: shared atomics from
# 20 warps, end-of-CTA flush by the last warp; storm mode without item lists),
# picked by the density feedback of the first launch on the handle (and
# forced); FLOW; the dynamic tail of the storm kernel (1.6 M records)
for n, dense in ((900_017, 0.05), (1_600_037, 0.02)):
    p = fpxgen.Params(seed=10, n_records=n, n_sites=40, recipe=fpxgen.RECIPE_STRESS, dense_nan=dense)
    hdr, arena, planes = fpxgen.generate_device(p)
    for mode, flags in ((0, 0), (0, fpx.OPT_STORM), (1, 0)):
        with fpx.Handle(0, flags=flags) as h:
            for _ in range(2):
                h.scan_records(hdr, arena, mode=mode, arena_planes=planes)
                torch.cuda.synchronize()  # the second launch reads the first one's feedback
            h.fetch()
# early notification ring (mapped host memory) and a shared (exported) table
with fpx.Handle(0, flags=fpx.OPT_LIVE_NEW) as h:
    h.export()
    h.scan_records(hdr, arena, arena_planes=planes)
    torch.cuda.synchronize()
    h.poll_new()
    h.fetch()
del hdr, arena
for dt in (torch.float32, torch.float64, torch.float16, torch.bfloat16):
    x = torch.randn(100_003, device=dev).to(dt)
    x[::997] = float("nan")
    with fpx.Handle(0) as h:
        for a in range(4):
            h.scan_tensor(x[a: x.numel() - a], site=a)
        h.fetch()
# fused multi-tensor scan: mixed formats, ragged heads / tails, an empty tensor
xs = [torch.randn(n, device=dev).to(dt) for n, dt in
      ((70_001, torch.float32), (0, torch.float16), (33_333, torch.bfloat16), (12_345, torch.float64))]
for i, x in enumerate(xs):
    if x.numel():
        x[i::501] = float("inf")
with fpx.Handle(0) as h:
    h.scan_tensors([(x[1:] if x.numel() > 1 else x, i, i << 20) for i, x in enumerate(xs)])
    h.fetch()
torch.cuda.synchronize()
print("sanitize workload ok")
