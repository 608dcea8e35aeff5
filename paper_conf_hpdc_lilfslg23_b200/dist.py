"""Multi-GPU: record-index sharding and the NCCL merge of per-GPU tables.

SURVEY §8(e): records are independent, so rank r of P scans the contiguous
range [floor(rN/P), floor((r+1)N/P)) with base_index = range start (first
indices are then global).  The only cross-rank state is the table, whose merge
is associative and commutative (key union, count sum, first-index min):

  1. fetch the local table on device, sorted by key      (fpx_table_fetch_device)
  2. all_gather the key counts, then the keys padded with EMPTY
  3. union = sort + unique of the gathered keys           (fpx_keys_unique_device)
  4. dense scatter: this rank's count / first per union key
     (0 / INT64_MAX when absent)                           (fpx_table_lookup_device)
  5. all_reduce SUM of counts, all_reduce MIN of firsts   (NCCL over NVLink)

Counts and first indices travel as int64 (first < 2^63; the absent sentinel
is INT64_MAX so a signed MIN is exact).  The collective plumbing below is
backend-agnostic so the same code runs under gloo on CPU in the tests, with
`ops` supplying the three table operations.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

KEY_EMPTY_I64 = -1  # 0xFFFFFFFFFFFFFFFF viewed as int64
FIRST_NONE = (1 << 63) - 1


def shard_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous record range of `rank` (floor(rN/P), floor((r+1)N/P))."""
    return (n * rank) // world, (n * (rank + 1)) // world


def merge(keys: torch.Tensor, counts: torch.Tensor, firsts: torch.Tensor, ops, group=None):
    """Merge this rank's sorted (keys, counts, firsts) with every other rank's.
    Returns the global (keys, counts, firsts), identical on all ranks.

    ops.unique(t) -> sorted unique keys of t without EMPTY
    ops.lookup(keys) -> (counts, firsts) of this rank's table for those keys
    """
    world = dist.get_world_size(group)
    dev = keys.device
    # NCCL moves device tensors over NVLink; gloo (CPU tests, or several
    # ranks sharing one GPU) needs host tensors
    comm = torch.device("cpu") if dist.get_backend(group) == "gloo" else dev
    n = torch.tensor([keys.numel()], dtype=torch.int64, device=comm)
    sizes = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(sizes, n, group=group)
    m = int(max(int(s.item()) for s in sizes))
    if m == 0:
        e = torch.empty(0, dtype=torch.int64, device=dev)
        return e, e.clone(), e.clone()
    padded = torch.full((m,), KEY_EMPTY_I64, dtype=torch.int64, device=comm)
    padded[: keys.numel()] = keys.to(comm)
    gathered = [torch.empty_like(padded) for _ in range(world)]
    dist.all_gather(gathered, padded, group=group)
    union = ops.unique(torch.cat(gathered).to(dev))
    c, f = ops.lookup(union)
    c, f = c.to(comm), f.to(comm)
    dist.all_reduce(c, op=dist.ReduceOp.SUM, group=group)
    dist.all_reduce(f, op=dist.ReduceOp.MIN, group=group)
    return union, c.to(dev), f.to(dev)


class DeviceOps:
    """The table operations of `merge`, run by libfpx.so kernels on the GPU."""

    def __init__(self, handle, stream=None):
        self.h = handle
        self.stream = stream

    def unique(self, t):
        return self.h.unique_device(t, stream=self.stream)

    def lookup(self, keys):
        return self.h.lookup_device(keys, stream=self.stream)


def merge_handle(handle, group=None, stream=None):
    """Fetch this rank's table on device and merge it across the group (NCCL)."""
    k, c, f = handle.fetch_device(stream=stream)
    return merge(k, c, f, DeviceOps(handle, stream), group=group)


class SharedTable:
    """Fused alternative to `merge` (SURVEY §8 e, NEXT): every rank scans into
    the home rank's device table through CUDA IPC peer mappings — the table
    updates (rare atomicCAS / Add / Min, only on exceptional warp-records) go
    over NVLink / NVSwitch inside the scan kernels, so there is no merge step.

        st = SharedTable(device)          # collective: home exports, others attach
        st.handle.scan_records(...)       # every rank, its own shard
        st.finish()                       # streams drained + barrier
        entries = st.fetch()              # home rank: the union table
    """

    def __init__(self, device: int, group=None, home: int = 0, **handle_kw):
        from . import fpx

        self.group, self.home = group, home
        self.rank = dist.get_rank(group)
        blob = [None]
        if self.rank == home:
            self.handle = fpx.Handle(device, **handle_kw)
            blob = [self.handle.export()]
        dist.broadcast_object_list(blob, src=home, group=group)
        err = None
        if self.rank != home:
            try:
                self.handle = fpx.Handle.attach(device, blob[0])
            except fpx.FpxError as e:  # e.g. no IPC / peer access between the GPUs
                self.handle, err = None, str(e)
        # collective verdict: every rank must be attached, else nobody uses it
        flags = [None] * dist.get_world_size(group)
        dist.all_gather_object(flags, err, group=group)
        self.error = next((f for f in flags if f is not None), None)
        if self.error is not None:
            if self.handle is not None and self.rank != home:
                self.handle.close()
            dist.barrier(group=group)
            if self.rank == home:
                self.handle.close()
            raise RuntimeError(f"shared table unavailable: {self.error}")

    # Ordering between ranks.  Under NCCL it is stream-ordered: a one-element
    # all_reduce enqueued on the scan stream completes on no rank before every
    # rank has reached it, so "home cleared the table" and "every rank's scan
    # finished" become device-side dependencies with no host round trip per
    # step.  Under gloo (CPU tests, ranks sharing one GPU) the host waits for
    # the stream and meets the other ranks at a barrier.
    def _sync(self, stream):
        s = torch.cuda.current_stream() if stream is None else stream
        if dist.get_backend(self.group) == "nccl":
            if getattr(self, "_tok", None) is None:
                self._tok = torch.zeros(1, dtype=torch.int32, device=torch.cuda.current_device())
            with torch.cuda.stream(s):
                dist.all_reduce(self._tok, group=self.group)
        else:
            s.synchronize()
            dist.barrier(group=self.group)

    def reset(self, stream=None):
        """Home clears the table; no rank scans again before the clear is done."""
        if self.rank == self.home:
            self.handle.reset(stream=stream)
        self._sync(stream)

    def finish(self, stream=None):
        """Every rank's inserts have landed in the home table: on return (gloo)
        or in `stream` order (NCCL; fetch() on the home rank waits for it)."""
        self._sync(stream)

    def fetch(self):
        assert self.rank == self.home, "the home rank owns the shared table"
        return self.handle.fetch()

    def close(self):
        dist.barrier(group=self.group)  # attached ranks unmap before the home frees
        if self.rank != self.home:
            self.handle.close()
        dist.barrier(group=self.group)
        if self.rank == self.home:
            self.handle.close()
