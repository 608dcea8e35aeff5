"""Parity of the CUDA path (through the C ABI) with the CPU oracle.

All integer outputs — keys, counts, first indices — must match bit for bit
after the library's sort by key (SURVEY §8 b/c).  Inputs are seeded synthetic
traces (fpxgen) and hand-built records; expectations come from the oracle or
from the closed-form aggregate of planted events, never from the GPU.
"""
import ctypes

import numpy as np
import pytest

import fpxgen
import oracle
from _records import (
    BF16, DEST, FLOW, FLOW_DETAIL, FP16, FP32, FP64, NAN, NONE, OP_FADD, Trace, describe_diff, entries_equal,
    expected_from_injections, load_worked_cases, table_dict,
)

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def fpx():
    from paper_conf_hpdc_lilfslg23_b200 import fpx as m

    return m


DEV = "cuda:0"


def to_dev(hdr, arena):
    d_hdr = torch.from_numpy(np.ascontiguousarray(hdr).view(np.int32).reshape(-1, 4)).to(DEV)
    a = np.ascontiguousarray(arena)
    if a.size == 0:
        a = np.zeros((1, 32), np.uint32)
    d_arena = torch.from_numpy(a.view(np.int32).reshape(-1)).to(DEV)
    return d_hdr, d_arena


def gpu_scan(fpx, hdr, arena, base=0, mode=DEST, **kw):
    d_hdr, d_arena = to_dev(hdr, arena)
    with fpx.Handle(0, **kw) as h:
        h.scan_records(d_hdr, d_arena, base_index=base, mode=mode, n_records=len(hdr),
                       arena_planes=arena.size // 32)
        ents = h.fetch()
        st = h.last_status
        stats = h.stats()
    return ents, st, stats


def oracle_scan(hdr, arena, base=0, mode=DEST):
    t = oracle.Table()
    t.scan_records(hdr, arena, base_index=base, mode=mode)
    return t


def assert_same(got, exp):
    assert entries_equal(got, exp), describe_diff(got, exp)


# ---------------------------------------------------------------------------
def test_worked_cases_gpu(fpx):
    tr = Trace(seed=4)
    cases = load_worked_cases()
    for i, c in enumerate(cases):
        dest = None if c["dest"] is None else int(c["dest"], 16)
        tr.add_value_record(site=100 + i, opclass=c["opclass"], fmt=c["fmt"], mask=0x8000_F00F, dest_bits=dest,
                            src_bits=[int(s, 16) for s in c["srcs"]])
    hdr, arena = tr.arrays()
    for mode, key in ((DEST, "expect_dest"), (FLOW, "expect_flow"), (FLOW_DETAIL, "expect_flow")):
        got, st, _ = gpu_scan(fpx, hdr, arena, base=5, mode=mode)
        assert st == fpx.OK
        assert_same(got, oracle_scan(hdr, arena, 5, mode).entries())
        d = table_dict(got)
        for i, c in enumerate(cases):
            mine = {k: v for k, v in d.items() if k[0] == 100 + i}
            if c[key] is None:
                assert not mine, c["name"]
            else:
                kind, flow = c[key]
                assert mine == {(100 + i, c["fmt"], flow, kind): [9, 5 + i]}, c["name"]
                det = [int(e["detail"]) for e in got if int(e["site"]) == 100 + i]
                assert det == [c["expect_detail"] if mode == FLOW_DETAIL else 0], c["name"]


def _brute_trace():
    from test_oracle_pins import _brute_records, _bits

    tr = Trace(seed=8)
    site = 0
    for fmt in (FP32, FP64):
        for op, dest, srcs in _brute_records(fmt):
            op2 = 5 if (fmt == FP64 and op == 4) else op
            tr.add_value_record(site, op2, fmt, 0xFFFFFFFF if site % 3 else 0x0F0F0F0F,
                                None if dest is None else _bits(fmt, dest), [_bits(fmt, s) for s in srcs])
            site += 1
    return tr.arrays()


@pytest.mark.parametrize("variant", [0, 1], ids=["tma", "ldg"])
@pytest.mark.parametrize("mode", [DEST, FLOW, FLOW_DETAIL])
def test_bruteforce_ieee_ops_gpu(fpx, mode, variant):
    hdr, arena = _brute_trace()
    got, st, _ = gpu_scan(fpx, hdr, arena, base=0, mode=mode, flags=variant)
    assert_same(got, oracle_scan(hdr, arena, 0, mode).entries())


# ---------------------------------------------------------------------------
RECIPES = [
    ("c1", fpxgen.RECIPE_C1, DEST, 100_000, 200),     # config C1 at full size
    ("mix", fpxgen.RECIPE_MIX, DEST, 200_003, 10_000),
    ("flow", fpxgen.RECIPE_FLOW, FLOW, 150_001, 1_000),
    ("flow_detail", fpxgen.RECIPE_FLOW, FLOW_DETAIL, 150_001, 1_000),
    ("flow_as_dest", fpxgen.RECIPE_FLOW, DEST, 50_017, 1_000),
    ("packed", fpxgen.RECIPE_PACKED, DEST, 120_007, 1_000),
]


@pytest.mark.parametrize("variant", [0, 1], ids=["tma", "ldg"])
@pytest.mark.parametrize("name,recipe,mode,n,sites", RECIPES, ids=[r[0] for r in RECIPES])
def test_synthetic_trace_parity(fpx, name, recipe, mode, n, sites, variant):
    p = fpxgen.Params(seed=0x5EED0000 + recipe, n_records=n, n_sites=sites, recipe=recipe, p_fp64=0.5)
    hdr, arena = fpxgen.generate_host(p)
    inj, w = fpxgen.plan_injections(p, 400, flow=(recipe == fpxgen.RECIPE_FLOW))
    fpxgen.apply_host(w, hdr, arena)
    base = 10**12 + 7
    got, st, stats = gpu_scan(fpx, hdr, arena, base=base, mode=mode, flags=variant)
    ref = oracle_scan(hdr, arena, base, mode)
    assert st == fpx.OK and stats.bad_records == 0
    assert_same(got, ref.entries())
    # and the independent closed form of the planted events (FLOW_DETAIL
    # splits entries further by source; its (site, fmt, flow, kind) sums match)
    if mode == FLOW_DETAIL:
        merged = {}
        for e in got:
            k = (int(e["site"]), int(e["fmt"]), int(e["flow"]), int(e["kind"]))
            c = merged.setdefault(k, [0, 2**64 - 1])
            c[0] += int(e["count"])
            c[1] = min(c[1], int(e["first_index"]))
        assert merged == expected_from_injections(hdr, inj, base, FLOW)
    else:
        assert table_dict(got) == expected_from_injections(hdr, inj, base, mode)


@pytest.mark.parametrize("variant", [0, 1, 2, 3, 8, 10],
                         ids=["tma", "ldg", "tma-noagg", "ldg-noagg", "tma-storm", "tma-storm-noagg"])
def test_dense_nan_storm(fpx, variant):
    p = fpxgen.Params(seed=77, n_records=60_000, n_sites=200, recipe=fpxgen.RECIPE_STRESS, dense_nan=1.0)
    hdr, arena = fpxgen.generate_host(p)
    got, st, _ = gpu_scan(fpx, hdr, arena, flags=variant)
    assert_same(got, oracle_scan(hdr, arena).entries())
    p.dense_nan = 0.01
    hdr, arena = fpxgen.generate_host(p)
    got, st, _ = gpu_scan(fpx, hdr, arena, base=3, flags=variant)
    assert_same(got, oracle_scan(hdr, arena, 3).entries())


@pytest.mark.parametrize("mode", [DEST, FLOW, FLOW_DETAIL], ids=["dest", "flow", "flow_detail"])
def test_no_warp_agg_ablation_same_table(fpx, mode):
    """FPX_OPT_NO_WARP_AGG (per-lane table updates) changes the cost, never the table."""
    recipe = fpxgen.RECIPE_MIX if mode == DEST else fpxgen.RECIPE_FLOW
    p = fpxgen.Params(seed=31 + mode, n_records=30_011, n_sites=50, recipe=recipe, p_partial=0.3)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 3000, flow=mode != DEST)
    fpxgen.apply_host(w, hdr, arena)
    exp = oracle_scan(hdr, arena, 11, mode).entries()
    for flags in (fpx.OPT_NO_WARP_AGG, fpx.OPT_NO_WARP_AGG | fpx.OPT_SCAN_LDG):
        got, st, _ = gpu_scan(fpx, hdr, arena, base=11, mode=mode, flags=flags)
        assert_same(got, exp)


@pytest.mark.parametrize("variant", [0, 1], ids=["tma", "ldg"])
@pytest.mark.parametrize("n", [1, 31, 32, 33, 255, 257, 4097])
def test_ragged_sizes(fpx, n, variant):
    p = fpxgen.Params(seed=n, n_records=n, n_sites=7, recipe=fpxgen.RECIPE_MIX, p_partial=0.5)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, max(1, n // 8))
    fpxgen.apply_host(w, hdr, arena)
    for mode in (DEST,):
        got, st, _ = gpu_scan(fpx, hdr, arena, base=n, mode=mode, flags=variant)
        assert_same(got, oracle_scan(hdr, arena, n, mode).entries())


def test_empty_scan_and_invalid_args(fpx):
    with fpx.Handle(0) as h:
        t = torch.zeros(16, dtype=torch.int32, device=DEV)
        assert fpx.lib.fpx_scan_records(h.ptr, t.data_ptr(), 0, t.data_ptr(), 0, 0, 0, None) == fpx.OK
        assert len(h.fetch()) == 0 and h.last_status == fpx.OK
        # misaligned header pointer, bad mode, NULL handle, bad fmt
        assert fpx.lib.fpx_scan_records(h.ptr, t.data_ptr() + 4, 1, t.data_ptr(), 1, 0, 0, None) == fpx.ERR_INVALID
        assert fpx.lib.fpx_scan_records(h.ptr, t.data_ptr(), 1, t.data_ptr(), 1, 0, 7, None) == fpx.ERR_INVALID
        assert fpx.lib.fpx_scan_records(None, t.data_ptr(), 1, t.data_ptr(), 1, 0, 0, None) == fpx.ERR_INVALID
        assert fpx.lib.fpx_scan_tensor(h.ptr, t.data_ptr(), 4, 9, 0, 0, None) == fpx.ERR_INVALID
        assert fpx.lib.fpx_scan_tensor(h.ptr, t.data_ptr() + 2, 4, FP32, 0, 0, None) == fpx.ERR_INVALID
    bad = ctypes.c_void_p()
    assert fpx.lib.fpx_open(0, ctypes.byref(fpx.Options(40, 0, 0)), ctypes.byref(bad)) == fpx.ERR_INVALID
    assert fpx.lib.fpx_open(99, None, ctypes.byref(bad)) == fpx.ERR_INVALID


def test_bad_records_sticky(fpx):
    tr = Trace()
    tr.add(3, OP_FADD, FP32, 0xFFFFFFFF, [0x7FC00000], [])
    tr.add(0xFFFFFFFF, OP_FADD, FP32, 0xFFFFFFFF, [0x7FC00000], [])
    tr.add(4, OP_FADD, FP32, 0xFFFFFFFF, [0x7FC00000], [])
    hdr, arena = tr.arrays()
    hdr[2]["meta"] |= 1 << 20
    got, st, stats = gpu_scan(fpx, hdr, arena)
    assert st == fpx.ERR_BAD_RECORD and stats.bad_records == 2
    assert_same(got, oracle_scan(hdr, arena).entries())
    # FLOW rejects packed records
    tr = Trace()
    tr.add(3, 15, FP16, 0xFFFFFFFF, [0x7C007C00], [])
    hdr, arena = tr.arrays()
    got, st, stats = gpu_scan(fpx, hdr, arena, mode=FLOW)
    assert st == fpx.ERR_BAD_RECORD and stats.bad_records == 1 and len(got) == 0


def test_table_full_drops_are_counted(fpx):
    # 64 distinct keys into a 16-slot table
    tr = Trace()
    for s in range(64):
        tr.add(s, OP_FADD, FP32, (1 << (s % 32)) | 1, [0x7FC00000], [])
    hdr, arena = tr.arrays()
    got, st, stats = gpu_scan(fpx, hdr, arena, table_log2_slots=4)
    ref = table_dict(oracle_scan(hdr, arena).entries())
    assert st == fpx.ERR_TABLE_FULL
    assert len(got) == 16 and stats.table_entries == 16
    d = table_dict(got)
    for k, v in d.items():
        assert ref[k] == v
    assert sum(v[0] for v in d.values()) + stats.dropped_events == sum(v[0] for v in ref.values())


def test_fetch_new_reports_only_new_keys(fpx):
    tr = Trace()
    tr.add(1, OP_FADD, FP32, 0xFFFFFFFF, [0x7FC00000], [])
    tr.add(2, OP_FADD, FP32, 0x1, [0x7F800000], [])
    h1, a1 = tr.arrays()
    tr.add(1, OP_FADD, FP32, 0x3, [0x7FC00000], [])  # existing key
    tr.add(9, OP_FADD, FP32, 0x1, [0x00000001], [])  # new key
    h2, a2 = tr.arrays()
    with fpx.Handle(0) as h:
        d1, da1 = to_dev(h1, a1)
        h.scan_records(d1, da1)
        new1 = h.fetch_new()
        assert table_dict(new1) == {(1, FP32, NONE, NAN): [32, 0], (2, FP32, NONE, 1): [1, 1]}
        d2, da2 = to_dev(h2[2:], a2)
        h.scan_records(d2, da2, base_index=2)
        new2 = h.fetch_new()
        assert table_dict(new2) == {(9, FP32, NONE, 2): [1, 3]}
        assert len(h.fetch_new()) == 0
        assert table_dict(h.fetch())[(1, FP32, NONE, NAN)] == [34, 0]


def test_streaming_batches_equal_single_scan(fpx):
    p = fpxgen.Params(seed=31, n_records=50_000, n_sites=300, recipe=fpxgen.RECIPE_MIX)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 200)
    fpxgen.apply_host(w, hdr, arena)
    d_hdr, d_arena = to_dev(hdr, arena)
    with fpx.Handle(0) as h:
        cuts = [0, 1, 4000, 4001, 33_333, 50_000]
        for a, b in zip(cuts, cuts[1:]):
            h.scan_records(d_hdr[a:b], d_arena, base_index=a, arena_planes=arena.size // 32)
        got = h.fetch()
    assert_same(got, oracle_scan(hdr, arena).entries())


# ---------------------------------------------------------------------------
# tensor scan
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("fmt", [FP16, BF16])
def test_tensor_exhaustive_16bit(fpx, fmt):
    bits = np.arange(65536, dtype=np.uint16)
    t = torch.from_numpy(bits.view(np.int16)).to(DEV)
    with fpx.Handle(0) as h:
        h.scan_tensor(t, fmt=fmt, site=3, base_index=100)
        got = h.fetch()
    ref = oracle.Table()
    ref.scan_tensor(bits, fmt, site=3, base_index=100)
    assert_same(got, ref.entries())
    counts = {int(e["kind"]): int(e["count"]) for e in got}
    assert counts == ({0: 2046, 1: 2, 2: 2046} if fmt == FP16 else {0: 254, 1: 2, 2: 254})


@pytest.mark.parametrize("fmt", [FP32, FP64, FP16, BF16])
@pytest.mark.parametrize("offset", [0, 1, 3, 7])
def test_tensor_misaligned_and_ragged(fpx, fmt, offset):
    dt = {FP32: np.uint32, FP64: np.uint64, FP16: np.uint16, BF16: np.uint16}[fmt]
    rng = np.random.default_rng(offset + 10 * fmt)
    n = 100_003
    bits = rng.integers(0, np.iinfo(dt).max, n + offset, dtype=dt, endpoint=True)
    t = torch.from_numpy(bits.view({1: np.int8, 2: np.int16, 4: np.int32, 8: np.int64}[bits.itemsize])).to(DEV)
    with fpx.Handle(0) as h:
        for k in range(3):  # a few sub-ranges, ragged on both ends
            a, b = offset + k, n + offset - 2 * k
            h.scan_tensor(t[a:b], fmt=fmt, site=k, base_index=a)
        got = h.fetch()
    ref = oracle.Table()
    for k in range(3):
        a, b = offset + k, n + offset - 2 * k
        ref.scan_tensor(bits[a:b], fmt, site=k, base_index=a)
    assert_same(got, ref.entries())


def test_tensor_exhaustive_fp32_closed_form(fpx):
    """All 2^32 FP32 bit patterns on the GPU, in 4 chunks of 2^30."""
    chunk = 1 << 30
    with fpx.Handle(0) as h:
        for c in range(4):
            t = (torch.arange(chunk, dtype=torch.int64, device=DEV) + c * chunk).to(torch.int32)
            h.scan_tensor(t, fmt=FP32, site=0, base_index=c * chunk)
            torch.cuda.synchronize()
            del t
        got = h.fetch()
    d = {int(e["kind"]): (int(e["count"]), int(e["first_index"])) for e in got}
    assert d == {0: (16_777_214, 0x7F800001), 1: (2, 0x7F800000), 2: (16_777_214, 1)}


def test_tensor_index_beyond_2_32(fpx):
    n = (1 << 32) + 1000
    t = torch.zeros(n, dtype=torch.float16, device=DEV)
    t[n - 5] = float("nan")
    t[7] = float("inf")
    with fpx.Handle(0) as h:
        h.scan_tensor(t, site=1, base_index=3)
        got = h.fetch()
    del t
    assert table_dict(got) == {(1, FP16, NONE, NAN): [1, 3 + n - 5], (1, FP16, NONE, 1): [1, 10]}


def test_tensor_torch_randn_with_planted(fpx):
    g = torch.Generator(device=DEV).manual_seed(5)
    for dtype, fmt in ((torch.float16, FP16), (torch.bfloat16, BF16), (torch.float32, FP32)):
        x = torch.randn(3_000_001, device=DEV, dtype=dtype, generator=g)
        x[::100_003] = float("nan")
        x[5::200_003] = float("-inf")
        x[17] = 0.0
        with fpx.Handle(0) as h:
            h.scan_tensor(x, site=2, base_index=0)
            got = h.fetch()
        host = x.view({2: torch.int16, 4: torch.int32}[x.element_size()]).cpu().numpy()
        ref = oracle.Table()
        ref.scan_tensor(host, fmt, site=2)
        assert_same(got, ref.entries())


# ---------------------------------------------------------------------------
# generator: device == host (the shared input module)
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("recipe", [fpxgen.RECIPE_MIX, fpxgen.RECIPE_FLOW, fpxgen.RECIPE_PACKED])
def test_generator_device_matches_host(recipe):
    p = fpxgen.Params(seed=99, n_records=20_011, n_sites=500, recipe=recipe)
    hdr, arena = fpxgen.generate_host(p, r0=12345)
    d_hdr, d_arena, planes = fpxgen.generate_device(p, r0=12345)
    assert planes == arena.shape[0]
    assert np.array_equal(d_hdr.cpu().numpy().view(np.uint32).reshape(-1), hdr.view(np.uint32).reshape(-1))
    assert np.array_equal(d_arena[: planes * 32].cpu().numpy().view(np.uint32), arena.reshape(-1))
    _, w = fpxgen.plan_injections(p, 100, r0=12345)
    fpxgen.apply_host(w, hdr, arena)
    fpxgen.apply_device(w, d_hdr, d_arena)
    assert np.array_equal(d_arena[: planes * 32].cpu().numpy().view(np.uint32), arena.reshape(-1))


@pytest.mark.parametrize("newlog_capacity", [0, 8])  # 8 < keys: the log overflows -> full clear
def test_reset_clears_every_key(fpx, newlog_capacity):
    p = fpxgen.Params(seed=3, n_records=30_000, n_sites=500, recipe=fpxgen.RECIPE_MIX)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 300)
    fpxgen.apply_host(w, hdr, arena)
    d_hdr, d_arena = to_dev(hdr, arena)
    ref = oracle_scan(hdr, arena).entries()
    with fpx.Handle(0, table_log2_slots=12, newlog_capacity=newlog_capacity) as h:
        for rep in range(3):
            h.scan_records(d_hdr, d_arena)
            got = h.fetch()
            assert_same(got, ref)
            st = h.stats()
            assert st.newlog_overflow == (0 if newlog_capacity == 0 else len(ref) - newlog_capacity)
            h.reset()
            assert len(h.fetch()) == 0 and h.stats().table_entries == 0


@pytest.mark.parametrize("mode", [DEST, FLOW, FLOW_DETAIL])
@pytest.mark.parametrize("n", [40_000, 1_700_003], ids=["static", "dynamic"])
def test_irregular_layouts(fpx, mode, n):
    """Producer layouts the generator never makes: records in shuffled arena
    order, several records sharing planes (broadcast immediates),
    records whose planes run past the arena (bad), DEST scans of records with
    sources (needed planes stop before the footprint ends); at a size that
    only uses static ranges and at one in the dynamic-tail regime."""
    p = fpxgen.Params(seed=17, n_records=n, n_sites=300, recipe=fpxgen.RECIPE_FLOW, p_fp64=0.4)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 400, flow=True)
    fpxgen.apply_host(w, hdr, arena)
    rng = np.random.default_rng(5)
    hdr2 = hdr.copy()
    perm = rng.permutation(len(hdr2))
    hdr2 = hdr2[perm]                                         # records no longer in arena order
    share = rng.choice(len(hdr2), 2000, replace=False)
    hdr2["val_off"][share[1000:]] = hdr2["val_off"][share[:1000]]  # pairs of records share planes
    hdr2["meta"][share[1000:]] = hdr2["meta"][share[:1000]]
    oob = rng.choice(len(hdr2), 50, replace=False)
    hdr2["val_off"][oob] = arena.shape[0] - 1                 # planes past the arena end -> bad records
    got, st, stats = gpu_scan(fpx, hdr2, arena, base=77, mode=mode)
    ref = oracle_scan(hdr2, arena, 77, mode)
    assert_same(got, ref.entries())
    assert stats.bad_records == ref.bad_records > 0


def test_scan_tensors_one_launch(fpx):
    """fpx_scan_tensors == one fpx_scan_tensor per descriptor == the oracle,
    over mixed formats, empty / tiny / misaligned / large tensors and a dense
    NaN tensor."""
    g = torch.Generator(device=DEV).manual_seed(11)
    items = []
    for i, (dt, n, off) in enumerate([(torch.float32, 0, 0), (torch.float16, 1, 0), (torch.bfloat16, 7, 3),
                                      (torch.float64, 1001, 1), (torch.float32, 100_003, 2), (torch.float16, 65_537, 5),
                                      (torch.bfloat16, 333_333, 0), (torch.float64, 12_345, 0), (torch.float32, 4096, 0)]):
        base = torch.randn(n + off, generator=g, device=DEV).to(dt)
        t = base[off:]
        if n > 10:
            t[:: max(1, n // 17)] = float("nan")
            t[5:: max(1, n // 7)] = float("-inf")
        if i == 8:
            t[:] = float("nan")  # dense
        items.append((t, 100 + i, 1000 * i))
    with fpx.Handle(0) as h:
        h.scan_tensors(items)
        got = h.fetch()
    with fpx.Handle(0) as h:
        for t, site, b in items:
            if t.numel():
                h.scan_tensor(t, site=site, base_index=b)
        single = h.fetch()
    ref = oracle.Table()
    for t, site, b in items:
        if t.numel():
            host = t.contiguous().view({2: torch.int16, 4: torch.int32, 8: torch.int64}[t.element_size()]).cpu().numpy()
            ref.scan_tensor(host, {torch.float32: FP32, torch.float64: FP64, torch.float16: FP16,
                                   torch.bfloat16: BF16}[t.dtype], site=site, base_index=b)
    assert_same(got, ref.entries())
    assert_same(single, ref.entries())


# ---------------------------------------------------------------------------
# Dynamic tail of the record scan (fpx_scan_records.cu Sched): from 16 tiles per
# warp up (148 * 20 * 512 = 1,515,520 records), warps scan 3/4 of the trace in
# static ranges and claim the rest: 256-record chunks, then 8 one-tile chunks
# per warp.  ~1.5e6 records: the rest fits the one-tile chunks alone; ~4e6:
# both kinds of chunk; the threshold itself and one record below it (static
# ranges only); ragged last chunks throughout.  The oracle finishes in seconds.
@pytest.mark.parametrize("name,recipe,mode,n", [
    ("mix", fpxgen.RECIPE_MIX, DEST, 1_600_037),
    ("flow", fpxgen.RECIPE_FLOW, FLOW, 1_550_011),
    ("packed", fpxgen.RECIPE_PACKED, DEST, 1_520_129),
    ("threshold", fpxgen.RECIPE_MIX, DEST, 1_515_520),
    ("below", fpxgen.RECIPE_MIX, DEST, 1_515_519),
    ("mix_big", fpxgen.RECIPE_MIX, DEST, 4_000_037),
    ("flow_big", fpxgen.RECIPE_FLOW, FLOW, 3_500_017),
    ("flow_detail", fpxgen.RECIPE_FLOW, FLOW_DETAIL, 1_600_001),
    ("mix_noagg", fpxgen.RECIPE_MIX, DEST, 1_700_011),
], ids=["mix", "flow", "packed", "threshold", "below", "mix_big", "flow_big", "flow_detail", "mix_noagg"])
def test_dynamic_tail_parity(fpx, name, recipe, mode, n):
    p = fpxgen.Params(seed=0x5EED0100 + recipe, n_records=n, n_sites=3_000, recipe=recipe, p_fp64=0.5)
    hdr, arena = fpxgen.generate_host(p)
    inj, w = fpxgen.plan_injections(p, 3_000, flow=(recipe == fpxgen.RECIPE_FLOW))
    fpxgen.apply_host(w, hdr, arena)
    base = 3 * 10**9
    flags = fpx.OPT_NO_WARP_AGG if name.endswith("noagg") else 0
    got, st, stats = gpu_scan(fpx, hdr, arena, base=base, mode=mode, flags=flags)
    assert st == fpx.OK and stats.bad_records == 0
    assert_same(got, oracle_scan(hdr, arena, base, mode).entries())
    if mode == FLOW_DETAIL:  # detail splits entries further; (site, fmt, flow, kind) sums match
        merged = {}
        for e in got:
            k = (int(e["site"]), int(e["fmt"]), int(e["flow"]), int(e["kind"]))
            c = merged.setdefault(k, [0, 2**64 - 1])
            c[0] += int(e["count"])
            c[1] = min(c[1], int(e["first_index"]))
        assert merged == expected_from_injections(hdr, inj, base, FLOW)
    else:
        assert table_dict(got) == expected_from_injections(hdr, inj, base, mode)


def test_dynamic_tail_relaunch_and_streams(fpx):
    """The chunk counters re-arm themselves: back-to-back launches without a
    reset add up exactly (count x 3, same first index), and launches in
    flight on two streams at once (different counter pairs) do too."""
    n = 1_600_001
    p = fpxgen.Params(seed=41, n_records=n, n_sites=500, recipe=fpxgen.RECIPE_MIX, p_fp64=0.5)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 2_000)
    fpxgen.apply_host(w, hdr, arena)
    exp = table_dict(oracle_scan(hdr, arena, 0, DEST).entries())
    d_hdr, d_arena = to_dev(hdr, arena)
    planes = arena.size // 32
    with fpx.Handle(0) as h:
        for _ in range(3):
            h.scan_records(d_hdr, d_arena, base_index=0, n_records=n, arena_planes=planes)
        got = table_dict(h.fetch())
        assert got == {k: [3 * c, f] for k, (c, f) in exp.items()}
        h.reset()
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        torch.cuda.synchronize()
        for _ in range(2):
            for s in (s1, s2):
                h.scan_records(d_hdr, d_arena, base_index=0, n_records=n, arena_planes=planes, stream=s)
        torch.cuda.synchronize()
        got = table_dict(h.fetch())
        assert got == {k: [4 * c, f] for k, (c, f) in exp.items()}


def test_scan_tensors_duplicate_sites_decreasing_bases_two_streams(fpx):
    """fpx_scan_tensors == the oracle when several descriptors share (site,
    fmt) with base indices in decreasing order (the merged event keeps the
    smaller first index), and when back-to-back calls on two streams reuse
    the library's descriptor buffer while the earlier launch may still run."""
    g = torch.Generator(device=DEV).manual_seed(3)
    items = []
    for i in range(12):
        t = torch.randn(50_000 + 37 * i, generator=g, device=DEV)
        t[(7 * i) % 1000] = float("nan")
        t[-1 - i] = float("inf")
        items.append((t, 5 + (i % 2), 10**9 - 10**6 * i))  # two sites, bases decreasing
    ref = oracle.Table()
    for t, site, b in items:
        ref.scan_tensor(t.view(torch.int32).cpu().numpy(), FP32, site=site, base_index=b)
    with fpx.Handle(0) as h:
        h.scan_tensors(items)
        got = h.fetch()
    assert_same(got, ref.entries())
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    with fpx.Handle(0) as h:
        for rep in range(20):  # alternate streams; each call rewrites the descriptor table
            h.scan_tensors(items[rep % 3::3], stream=s1 if rep % 2 else s2)
        torch.cuda.synchronize()
        got = table_dict(h.fetch())
    exp = {}
    for rep in range(20):
        for t, site, b in items[rep % 3::3]:
            r = oracle.Table()
            r.scan_tensor(t.view(torch.int32).cpu().numpy(), FP32, site=site, base_index=b)
            for k, (c, f) in table_dict(r.entries()).items():
                e = exp.setdefault(k, [0, 2**64 - 1])
                e[0] += c
                e[1] = min(e[1], f)
    assert got == exp


def test_fetch_new_truncated_windows_lose_nothing(fpx):
    tr = Trace()
    for s in range(100):
        tr.add(s, OP_FADD, FP32, 0x1, [0x7FC00000], [])
    hdr, arena = tr.arrays()
    d_hdr, d_arena = to_dev(hdr, arena)
    with fpx.Handle(0) as h:
        h.scan_records(d_hdr, d_arena)
        seen = []
        while True:
            part = h.fetch_new(capacity=30)
            if len(part) == 0:
                break
            assert h.last_status in (fpx.OK, fpx.ERR_TRUNCATED)
            seen += [int(e["site"]) for e in part]
        assert sorted(seen) == list(range(100))  # each new key exactly once
        with pytest.raises(ValueError):
            h.fetch(flags=fpx.FETCH_NEW)
        tr2 = Trace()
        tr2.add(500, OP_FADD, FP32, 0x1, [0x7F800000], [])
        h2, a2 = tr2.arrays()
        d2, da2 = to_dev(h2, a2)
        h.scan_records(d2, da2)
        assert [int(e["site"]) for e in h.fetch_new(capacity=30)] == [500]


@pytest.mark.parametrize("dense", [1.0, 0.01])
def test_storm_cta_large_launch(fpx, dense):
    """A storm launch of more than 2^24 records: the CTA table then adds its
    counts with the returning atomic and drains a slot before 2^31 (below
    2^24 records it uses a shared reduction, which cannot overflow there);
    the table must still equal the oracle's."""
    n = (1 << 24) + 4099
    p = fpxgen.Params(seed=90, n_records=n, n_sites=200, recipe=fpxgen.RECIPE_STRESS, dense_nan=dense)
    hdr, arena = fpxgen.generate_host(p)
    base = 11
    exp = oracle_scan(hdr, arena, base, DEST).entries()
    got, st, _ = gpu_scan(fpx, hdr, arena, base=base, mode=DEST, flags=fpx.OPT_STORM)
    assert st == fpx.OK
    assert_same(got, exp)


@pytest.mark.parametrize("mode", [DEST, FLOW, FLOW_DETAIL])
@pytest.mark.parametrize("dense", [1.0, 0.01])
def test_storm_cta_preaggregation(fpx, mode, dense):
    """Storms long enough for warps to warm up the CTA pre-aggregation table
    (> 8 hit tiles per warp: 1.6e6 records on 2960 warps; the dynamic tail
    publishes the density that picks the storm kernel) and dense tiles
    (>= 4 records with events): the table equals the oracle's, so the
    shared-memory counts, the first-sighting inserts and the end-of-CTA flush
    add up exactly; and equals the per-lane ablation."""
    p = fpxgen.Params(seed=88, n_records=1_600_001, n_sites=200, recipe=fpxgen.RECIPE_STRESS, dense_nan=dense)
    hdr, arena = fpxgen.generate_host(p)
    base = 7 * 10**9
    exp = oracle_scan(hdr, arena, base, mode).entries()
    for flags in (0, fpx.OPT_STORM, fpx.OPT_NO_WARP_AGG):
        got, st, _ = gpu_scan(fpx, hdr, arena, base=base, mode=mode, flags=flags)
        assert st == fpx.OK
        assert_same(got, exp)
    # adaptive kernel choice: the handle's first scan uses the sparse kernel,
    # the density it reports switches the next ones to the storm kernel; and
    # a sparse trace scanned after the storm is still exact
    d_hdr, d_arena = to_dev(hdr, arena)
    q = fpxgen.Params(seed=89, n_records=1_600_013, n_sites=500, recipe=fpxgen.RECIPE_MIX, p_fp64=0.5)
    qh, qa = fpxgen.generate_host(q)
    _, w = fpxgen.plan_injections(q, 500)
    fpxgen.apply_host(w, qh, qa)
    q_exp = oracle_scan(qh, qa, 5, DEST).entries()
    dq_hdr, dq_arena = to_dev(qh, qa)
    with fpx.Handle(0) as h:
        for rep in range(3):
            h.scan_records(d_hdr, d_arena, base_index=base, mode=mode, arena_planes=arena.shape[0])
            assert_same(h.fetch(), exp)
            h.reset()
        for rep in range(2):
            h.scan_records(dq_hdr, dq_arena, base_index=5, arena_planes=qa.shape[0])
            assert_same(h.fetch(), q_exp)
            h.reset()
