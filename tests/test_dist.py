"""Multi-GPU merge logic (SURVEY §8 e) under gloo on CPU, world size 2 and 3.

Each rank scans its contiguous record shard (base_index = shard start) — here
with the CPU oracle standing in for a GPU table, since this container has no
GPU — and the shards are merged by paper_conf_hpdc_lilfslg23_b200.dist.merge
(all_gather of sizes and EMPTY-padded keys, union, dense scatter, all_reduce
SUM / MIN).  The merged table must equal a single scan of the whole trace.
A GPU version of the same check runs in tests/test_gpu_fullsize.py with the
library's device ops.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import fpxgen
import oracle


class CpuOps:
    """The three table operations of dist.merge over a Python dict table."""

    def __init__(self, table: dict):
        self.t = table

    def unique(self, keys):
        k = keys[keys != -1]
        u = np.unique(k.numpy().view(np.uint64))
        return torch.from_numpy(u.view(np.int64).copy())

    def lookup(self, keys):
        c = torch.zeros_like(keys)
        f = torch.full_like(keys, (1 << 63) - 1)
        for i, k in enumerate(keys.tolist()):
            if k in self.t:
                c[i], f[i] = self.t[k]
        return c, f


def _key(e):
    k = (int(e["site"]) << 32) | (int(e["fmt"]) << 4) | (int(e["flow"]) << 2) | int(e["kind"])
    return k - (1 << 64) if k >= (1 << 63) else k


def _worker(rank, world, port, n, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_hpdc_lilfslg23_b200 import dist as fdist

    p = fpxgen.Params(seed=42, n_records=n, n_sites=50, recipe=fpxgen.RECIPE_MIX)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 300)
    fpxgen.apply_host(w, hdr, arena)
    a, b = fdist.shard_range(n, rank, world)
    t = oracle.Table()
    t.scan_records(hdr[a:b], arena, base_index=a)
    ents = t.entries()
    local = {_key(e): (int(e["count"]), int(e["first_index"])) for e in ents}
    keys = torch.tensor(sorted(local), dtype=torch.int64)
    cnt = torch.tensor([local[k][0] for k in sorted(local)], dtype=torch.int64)
    fst = torch.tensor([local[k][1] for k in sorted(local)], dtype=torch.int64)
    u, c, f = fdist.merge(keys, cnt, fst, CpuOps(local))
    out_q.put((rank, u.tolist(), c.tolist(), f.tolist()))
    dist.barrier()
    dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_merge_equals_single_scan(world):
    n = 6007
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    results = [q.get(timeout=120) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    # every rank holds the same merged table ...
    merged = {r: {k: (c, f) for k, c, f in zip(u, cs, fs)} for r, u, cs, fs in results}
    assert all(merged[r] == merged[0] for r in merged)
    # ... equal to one scan of the whole trace
    p = fpxgen.Params(seed=42, n_records=n, n_sites=50, recipe=fpxgen.RECIPE_MIX)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 300)
    fpxgen.apply_host(w, hdr, arena)
    t = oracle.Table()
    t.scan_records(hdr, arena)
    ref = {_key(e): (int(e["count"]), int(e["first_index"])) for e in t.entries()}
    assert merged[0] == ref
    assert len(ref) > 20


def test_shard_ranges_cover_exactly():
    from paper_conf_hpdc_lilfslg23_b200 import dist as fdist

    for n in (0, 1, 7, 1000, 10**11):
        for world in (1, 2, 3, 8):
            rs = [fdist.shard_range(n, r, world) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(world - 1))
            assert max(b - a for a, b in rs) - min(b - a for a, b in rs) <= 1
