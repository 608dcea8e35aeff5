"""Mixed-code parity: per-lane independent special values, every opclass.

The GPU tables (through the C ABI) must equal the oracle's entry by entry on
"zoo" traces (tests/_mixed.py) where one warp-record holds several (kind,
flow) codes at once — Alg2's leader loop over lanes with different exceptions
 — in DEST, FLOW and FLOW_DETAIL, on both record kernels, with and
without warp aggregation; at a size that uses static ranges only and at one
in the dynamic-tail regime.  The fast path's witness check is tested for
false negatives with one exceptional candidate per tile: every exceptional
FP16 / BF16 half in the low and high position of the packed word next to
halves of both signs, and the FP32 / FP64 boundary sets.
"""
import numpy as np
import pytest

import oracle
from _mixed import isolated_fp64_trace, isolated_word_trace, sparse_flow_trace, zoo_trace
from _records import (
    BF16, DEST, FLOW, FLOW_DETAIL, FP16, FP32, FP64, NONE, describe_diff, entries_equal, np_class, table_dict,
)

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
DEV = "cuda:0"
KIND = {1: 0, 2: 1, 3: 2}  # np_class code -> E_exce kind


@pytest.fixture(scope="module")
def fpx():
    from paper_conf_hpdc_lilfslg23_b200 import fpx as m

    return m


def to_dev(hdr, arena):
    d_hdr = torch.from_numpy(np.ascontiguousarray(hdr).view(np.int32).reshape(-1, 4)).to(DEV)
    a = np.ascontiguousarray(arena)
    if a.size == 0:
        a = np.zeros((1, 32), np.uint32)
    return d_hdr, torch.from_numpy(a.view(np.int32).reshape(-1)).to(DEV)


def gpu_table(fpx, hdr, arena, base, mode, flags):
    d_hdr, d_arena = to_dev(hdr, arena)
    with fpx.Handle(0, flags=flags) as h:
        h.scan_records(d_hdr, d_arena, base_index=base, mode=mode, n_records=len(hdr), arena_planes=arena.shape[0])
        got = h.fetch()
        stats = h.stats()
    return got, stats


_cache = {}


def _trace(n, flow):
    k = (n, flow)
    if k not in _cache:
        _cache.clear()
        hdr, arena = zoo_trace(seed=1000 + n + flow, n=n, flow=flow)
        _cache[k] = (hdr, arena, {})
    return _cache[k]


def _oracle(n, flow, mode, base):
    hdr, arena, exp = _trace(n, flow)
    if mode not in exp:
        t = oracle.Table()
        t.scan_records(hdr, arena, base_index=base, mode=mode)
        exp[mode] = (t.entries(), t.bad_records)
    return exp[mode]


VARIANTS = [(0, "tma"), (1, "ldg"), (2, "tma-noagg"), (3, "ldg-noagg"), (8, "tma-storm"), (10, "tma-storm-noagg")]


@pytest.mark.parametrize("n", [50_011, 1_600_037], ids=["static", "dynamic"])
@pytest.mark.parametrize("mode", [DEST, FLOW, FLOW_DETAIL], ids=["dest", "flow", "flow_detail"])
@pytest.mark.parametrize("flags", [v[0] for v in VARIANTS], ids=[v[1] for v in VARIANTS])
def test_zoo_parity(fpx, n, mode, flags):
    hdr, arena, _ = _trace(n, mode != DEST)
    base = 5 * 10**9 + 3
    exp, bad = _oracle(n, mode != DEST, mode, base)
    got, stats = gpu_table(fpx, hdr, arena, base, mode, flags)
    assert entries_equal(got, exp), describe_diff(got, exp)
    assert stats.bad_records == bad
    assert (bad > 0) == (mode != DEST)  # FLOW modes reject the packed records (R13)
    # the trace really mixes codes: many keys per site, every kind and flow
    kinds = {int(e["kind"]) for e in exp}
    flows = {int(e["flow"]) for e in exp}
    assert kinds == {0, 1, 2, 3}
    assert flows == ({NONE} if mode == DEST else {1, 2, 3})
    if mode == FLOW_DETAIL:
        assert {int(e["detail"]) for e in exp} >= {0, 1, 2, 3, 5, 6, 7}


@pytest.mark.parametrize("n", [200_003, 1_600_037], ids=["static", "dynamic"])
@pytest.mark.parametrize("mode", [FLOW, FLOW_DETAIL], ids=["flow", "flow_detail"])
@pytest.mark.parametrize("flags", [0, 1], ids=["tma", "ldg"])
def test_flow_sparse_candidates(fpx, n, mode, flags):
    """Hit analyzer tiles with one or two exceptional records among clean
    ones: the exact path walks only the records with a candidate plane
    (flow_candidates); the table must still equal the oracle's."""
    hdr, arena = sparse_flow_trace(seed=77 + n, n=n)
    base = 12345
    t = oracle.Table()
    t.scan_records(hdr, arena, base_index=base, mode=mode)
    exp = t.entries()
    got, stats = gpu_table(fpx, hdr, arena, base, mode, flags)
    assert entries_equal(got, exp), describe_diff(got, exp)
    assert stats.bad_records == t.bad_records
    assert {int(e["flow"]) for e in exp} == {1, 2, 3}
    # sparse: far fewer events than records
    assert int(np.sum(exp["count"])) < n // 4


# ---------------------------------------------------------------------------
# witness isolation: one exceptional candidate per tile (no false negatives)
# ---------------------------------------------------------------------------
def _closed_form(carrier_fmt, values, sites, first_of):
    """Expected table of an isolation trace from numpy's IEEE predicates."""
    cls = np_class(carrier_fmt, values.astype(np.uint64))
    exp = {}
    for t, c in enumerate(cls):
        if c:
            e = exp.setdefault((int(sites[t]), carrier_fmt, NONE, KIND[int(c)]), [0, first_of(t)])
            e[0] += 1
    return exp


def _half_candidates(fmt):
    allv = np.arange(65536, dtype=np.uint64)
    exc = allv[np_class(fmt, allv) != 0]
    one = 0x3C00 if fmt == FP16 else 0x3F80
    words, halves = [], []
    for nb in (0x0000, 0x8000, one, one | 0x8000):  # neighbours of both signs (the doubling's carry)
        words.append(exc | (np.uint64(nb) << np.uint64(16)))  # candidate in the low half
        halves.append(exc)
        words.append((exc << np.uint64(16)) | np.uint64(nb))  # candidate in the high half
        halves.append(exc)
    return np.concatenate(words), np.concatenate(halves)


@pytest.mark.parametrize("flags", [0, 1], ids=["tma", "ldg"])
@pytest.mark.parametrize("fmt", [FP16, BF16])
def test_witness_every_exceptional_half_alone_in_its_tile(fpx, fmt, flags):
    words, halves = _half_candidates(fmt)
    one = 0x3C00 if fmt == FP16 else 0x3F80
    hdr, arena = isolated_word_trace(words, opclass=15, fmt=fmt, filler=one | (one << 16))
    got, stats = gpu_table(fpx, hdr, arena, 0, DEST, flags)
    exp = _closed_form(fmt, halves, np.arange(len(words)) % 7, lambda t: 32 * t)
    assert table_dict(got) == exp
    assert sum(v[0] for v in exp.values()) == len(words)  # every candidate exceptional
    ref = oracle.Table()
    ref.scan_records(hdr, arena)
    assert entries_equal(got, ref.entries()), describe_diff(got, ref.entries())


@pytest.mark.parametrize("flags", [0, 1], ids=["tma", "ldg"])
@pytest.mark.parametrize("fmt", [FP16, BF16])
def test_all_halves_both_positions_dense(fpx, fmt, flags):
    """All 2^16 halves (clean ones too) in both positions of the word next to
    +-0 and +-1 neighbours, packed densely: parity with the oracle."""
    allv = np.arange(65536, dtype=np.uint64)
    one = 0x3C00 if fmt == FP16 else 0x3F80
    w = np.concatenate([np.concatenate([allv | np.uint64(nb << 16), (allv << np.uint64(16)) | np.uint64(nb)])
                        for nb in (0, 0x8000, one, one | 0x8000)]).astype(np.uint32)
    from _records import HDR_DTYPE, meta

    n = len(w) // 32
    hdr = np.zeros(n, dtype=HDR_DTYPE)
    hdr["site"] = np.arange(n) % 3
    hdr["meta"] = meta(15, fmt, 0, 1)
    hdr["val_off"] = np.arange(n)
    hdr["active_mask"] = 0xFFFFFFFF
    arena = w.reshape(n, 32)
    got, _ = gpu_table(fpx, hdr, arena, 9, DEST, flags)
    ref = oracle.Table()
    ref.scan_records(hdr, arena, base_index=9)
    assert entries_equal(got, ref.entries()), describe_diff(got, ref.entries())


def _fp32_boundary():
    mags = [0, 1, 2, 0x3FFFFF, 0x400000, 0x7FFFFE, 0x7FFFFF, 0x800000, 0x800001, 0x7F7FFFFE, 0x7F7FFFFF,
            0x7F800000, 0x7F800001, 0x7F800002, 0x7FBFFFFF, 0x7FC00000, 0x7FC00001, 0x7FFFFFFE, 0x7FFFFFFF]
    return np.array(mags + [m | 0x80000000 for m in mags], dtype=np.uint64)


def _fp64_boundary():
    his = [0x00000000, 0x00000001, 0x000FFFFF, 0x00100000, 0x00100001, 0x7FEFFFFF, 0x7FF00000, 0x7FF00001,
           0x7FF7FFFF, 0x7FF80000, 0x7FFFFFFF]
    los = [0x00000000, 0x00000001, 0x80000000, 0xFFFFFFFF]
    v = [(h << 32) | l for h in his for l in los]
    return np.array(v + [x | (1 << 63) for x in v], dtype=np.uint64)


@pytest.mark.parametrize("flags", [0, 1], ids=["tma", "ldg"])
def test_witness_fp32_fp64_boundaries_alone_in_their_tiles(fpx, flags):
    v32 = _fp32_boundary()
    hdr, arena = isolated_word_trace(v32, opclass=1, fmt=FP32, filler=0x3F800000)
    got, _ = gpu_table(fpx, hdr, arena, 0, DEST, flags)
    assert table_dict(got) == _closed_form(FP32, v32, np.arange(len(v32)) % 7, lambda t: 32 * t)
    v64 = _fp64_boundary()
    hdr, arena = isolated_fp64_trace(v64)
    got, _ = gpu_table(fpx, hdr, arena, 0, DEST, flags)
    exp = _closed_form(FP64, v64, np.arange(len(v64)) % 5, lambda t: 80 * t)
    assert table_dict(got) == exp and len(exp) >= 3
