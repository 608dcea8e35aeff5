"""Count the kernels one NCCL/gloo merge step launches (for bench.py's
gpu_launches claim at N > 1): run under `ncu --metrics gpu__time_duration.sum`
with a world-size-1 gloo group on one GPU."""
import os
import sys

import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import fpxgen  # noqa: E402
from paper_conf_hpdc_lilfslg23_b200 import dist as fdist  # noqa: E402
from paper_conf_hpdc_lilfslg23_b200 import fpx  # noqa: E402

os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
os.environ.setdefault("MASTER_PORT", "29517")
dist.init_process_group("gloo", rank=0, world_size=1)
p = fpxgen.Params(seed=1, n_records=1_000_000, n_sites=10_000, recipe=fpxgen.RECIPE_MIX)
hdr, arena, planes = fpxgen.generate_device(p)
_, w = fpxgen.plan_injections(p, int(1e-6 * 32 * 1_000_000) + 200)
fpxgen.apply_device(w, hdr, arena)
h = fpx.Handle(0)
h.scan_records(hdr, arena, arena_planes=planes)
torch.cuda.synchronize()
torch.cuda.nvtx.range_push("merge")
k, c, f = fdist.merge_handle(h)
torch.cuda.synchronize()
torch.cuda.nvtx.range_pop()
print("merged keys", len(k))
dist.destroy_process_group()
