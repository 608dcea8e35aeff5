"""Pins of the CPU oracle against what the paper and the mathematics fix.

Each test pins the oracle to something other than itself:
  * closed-form counts of IEEE special values over exhaustive bit patterns
    (FP16 / BF16 all 2^16, FP32 all 2^32) — §2.1 P:140-145;
  * numpy's own IEEE predicates (a library routine) on boundary sets;
  * the paper's worked cases (tests/golden/worked_cases.json, each cited);
  * real IEEE arithmetic (numpy ops) brute-forced over special operands;
  * pure-Python brute force over tiny traces;
  * the closed-form aggregate of planted events in synthetic traces.
"""
import itertools

import numpy as np
import pytest

import fpxgen
import oracle
from _records import (
    BF16, DEST, DIV0, FLOW, FLOW_DETAIL, FP16, FP32, FP64, GEN, INF, KILL, NAN, NONE, OP_DIV, OP_DSETP, OP_FADD,
    OP_FFMA, OP_FMNMX, OP_FMUL, OP_FSEL, OP_FSET, OP_FSETP, OP_RCP, OP_RCP64H, PROP, SUB, Trace, expected_from_injections,
    load_worked_cases, np_class, table_dict, words_of,
)

CLEAN, C_NAN, C_INF, C_SUB = 0, 1, 2, 3


# --------------------------------------------------------------------------
# classification (a2): exhaustive closed forms and a library cross-check
# --------------------------------------------------------------------------
@pytest.mark.parametrize(
    "fmt,expected",
    [
        # 5-bit exponent, 10-bit mantissa: NaN = 2*(2^10-1), INF = 2, SUB = 2*(2^10-1), zero = 2
        (FP16, {C_NAN: 2046, C_INF: 2, C_SUB: 2046, CLEAN: 65536 - 2046 - 2 - 2046}),
        # 8-bit exponent, 7-bit mantissa
        (BF16, {C_NAN: 254, C_INF: 2, C_SUB: 254, CLEAN: 65536 - 254 - 2 - 254}),
    ],
)
def test_exhaustive_16bit_closed_form(fmt, expected):
    t = oracle.Table()
    bits = np.arange(65536, dtype=np.uint16)
    t.scan_tensor(bits, fmt, site=5)
    got = {int(e["kind"]): int(e["count"]) for e in t.entries()}
    assert got == {NAN: expected[C_NAN], INF: expected[C_INF], SUB: expected[C_SUB]}
    # element-wise against numpy's IEEE predicates
    cls = np.array([oracle.classify(fmt, int(b)) for b in range(65536)])
    assert np.array_equal(cls, np_class(fmt, bits.astype(np.uint64)))
    assert (cls == CLEAN).sum() == expected[CLEAN]


def test_exhaustive_fp32_closed_form():
    # all 2^32 patterns: NaN = SUB = 2*(2^23-1), INF = 2, zero = 2
    c = oracle.class_hist_fp32(0, 0xFFFFFFFF)
    assert int(c[C_NAN]) == 16_777_214
    assert int(c[C_INF]) == 2
    assert int(c[C_SUB]) == 16_777_214
    assert int(c[CLEAN]) == 2**32 - 2 * 16_777_214 - 2


def test_fp32_boundaries_and_random_vs_numpy():
    rng = np.random.default_rng(1)
    b = [0, 1, 0x7FFFFF, 0x800000, 0x7F7FFFFF, 0x7F800000, 0x7F800001, 0x7FC00000, 0x7FFFFFFF]
    b += [x | 0x80000000 for x in b]
    b += list(rng.integers(0, 2**32, 20000, dtype=np.uint64))
    b = np.array(b, dtype=np.uint64)
    got = np.array([oracle.classify(FP32, int(x)) for x in b])
    assert np.array_equal(got, np_class(FP32, b))


def test_fp64_boundaries_vs_numpy():
    base = [
        0x0000000000000001, 0x000FFFFFFFFFFFFF, 0x0010000000000000, 0x7FEFFFFFFFFFFFFF,
        0x7FF0000000000000, 0x7FF0000000000001, 0x7FF0000100000000, 0x7FF8000000000000,
        0x0000000100000000, 0x0000000000000000, 0x3FF0000000000000,
    ]
    b = base + [x | 0x8000000000000000 for x in base]
    rng = np.random.default_rng(2)
    b += [int(x) for x in rng.integers(0, 2**63, 20000, dtype=np.uint64)]
    b = np.array(b, dtype=np.uint64)
    got = np.array([oracle.classify(FP64, int(x)) for x in b])
    assert np.array_equal(got, np_class(FP64, b))
    # the two one-word traps
    assert oracle.classify(FP64, 0x7FF0000000000001) == C_NAN
    assert oracle.classify(FP64, 0x0000000100000000) == C_SUB


# --------------------------------------------------------------------------
# kind rule + flow rule: the paper's worked cases (golden fixtures)
# --------------------------------------------------------------------------
def _run_case(case, mode):
    fmt = case["fmt"]
    dest = None if case["dest"] is None else int(case["dest"], 16)
    srcs = [int(s, 16) for s in case["srcs"]]
    tr = Trace(seed=3)
    mask = 0b1000_0000_0000_0000_0000_0000_0100_1011  # 5 active lanes; the rest hold garbage
    r = tr.add_value_record(site=77, opclass=case["opclass"], fmt=fmt, mask=mask, dest_bits=dest, src_bits=srcs)
    hdr, arena = tr.arrays()
    t = oracle.Table()
    t.scan_records(hdr, arena, base_index=1000, mode=mode)
    assert t.bad_records == 0
    return t.entries(), r


@pytest.mark.parametrize("case", load_worked_cases(), ids=lambda c: c["name"])
def test_worked_case(case):
    for mode, key in ((DEST, "expect_dest"), (FLOW, "expect_flow"), (FLOW_DETAIL, "expect_flow")):
        ents, r = _run_case(case, mode)
        exp = case[key]
        if exp is None:
            assert len(ents) == 0, (mode, ents)
        else:
            assert len(ents) == 1, (mode, ents)
            e = ents[0]
            assert (int(e["kind"]), int(e["flow"])) == tuple(exp), (mode, e)
            assert int(e["site"]) == 77 and int(e["fmt"]) == case["fmt"]
            assert int(e["count"]) == 5 and int(e["first_index"]) == 1000 + r
            assert int(e["detail"]) == (case["expect_detail"] if mode == FLOW_DETAIL else 0), (mode, e)


# --------------------------------------------------------------------------
# brute force: special operands through real IEEE ops (numpy), both formats
# --------------------------------------------------------------------------
def _specials(fmt):
    if fmt == FP32:
        f = np.float32
        sub = np.array([0x00000123], dtype=np.uint32).view(np.float32)[0]
    else:
        f = np.float64
        sub = np.array([0x0000000000000123], dtype=np.uint64).view(np.float64)[0]
    return [f(0.0), f(-0.0), f(1.5), sub, f(np.inf), f(-np.inf), f(np.nan)]


def _bits(fmt, x):
    return int(np.array([x]).view(np.uint32 if fmt == FP32 else np.uint64)[0])


def _ieee_expect(fmt, op, dest, srcs):
    """(dest kind, flow-mode (kind, flow)) from numpy's IEEE predicates and the
    Table 2 states.  dest=None: no FP destination."""
    cls = lambda v: int(np_class(fmt, np.array([_bits(fmt, v)], dtype=np.uint64))[0])
    kind = {C_NAN: NAN, C_INF: INF, C_SUB: SUB}
    D = None
    if dest is not None and op != OP_FSET:  # FSET's destination is an integer mask (R10)
        cd = cls(dest)
        if op in (OP_RCP, OP_RCP64H):
            D = DIV0 if cd in (C_NAN, C_INF) else None
        elif op == OP_DIV and srcs[1] == 0 and np.isfinite(srcs[0]) and srcs[0] != 0:
            D = DIV0
        else:
            D = kind.get(cd)
    sev = {C_NAN: 3, C_INF: 2, C_SUB: 1, CLEAN: 0}
    S = max((cls(s) for s in srcs), key=lambda c: sev[c])
    S = kind.get(S) if sev[S] else None
    if D is not None and S is None:
        fl = (D, GEN)
    elif D is not None:
        fl = (D, PROP)
    elif S is not None:
        fl = (S, KILL)
    else:
        fl = None
    # FLOW_DETAIL: 1 + lowest index of a source with the most severe class,
    # | 4 for Table 1's control-flow opcodes (Table 2 "Comparison")
    det = 0
    if S is not None:
        classes = [cls(s) for s in srcs]
        det = 1 + next(i for i, c in enumerate(classes) if sev[c] == max(sev[x] for x in classes))
        if op in (OP_FSEL, OP_FSET, OP_FSETP, OP_FMNMX, OP_DSETP):  # Table 1's right column
            det |= 4
    return (None if D is None else (D, NONE)), fl, det


def _brute_records(fmt):
    sp = _specials(fmt)
    ftype = type(sp[0])
    cases = []
    with np.errstate(all="ignore"):
        for a, b in itertools.product(sp, sp):
            cases.append((OP_FADD, a + b, [a, b]))
            cases.append((OP_FMUL, a * b, [a, b]))
            cases.append((OP_DIV, a / b, [a, b]))
            cases.append((OP_FMNMX, np.fmin(a, b), [a, b]))  # IEEE-2008 minNum
            # compare-and-set predicate (FSETP / DSETP, T1 P:101-110): no FP destination
            cases.append((OP_FSETP if fmt == FP32 else OP_DSETP, None, [a, b]))
            if fmt == FP32:
                # FSET (T1: FP32 Compare And Set) writes the integer mask of a < b:
                # 0xFFFFFFFF when true -- a NaN bit pattern that is not a NaN (R10)
                cases.append((OP_FSET, np.array([0xFFFFFFFF if a < b else 0], np.uint32).view(np.float32)[0], [a, b]))
            cases.append((OP_FSEL, a, [a, b]))  # predicate true: selects a
            cases.append((OP_FSEL, b, [a, b]))  # predicate false: selects b
        for a, b, c in itertools.product(sp, sp, sp):
            cases.append((OP_FFMA, ftype(a * b + c) if fmt == FP64 else np.float32(np.float64(a) * np.float64(b) + np.float64(c)), [a, b, c]))
        for a in sp:
            cases.append((OP_RCP, ftype(1) / a, [a]))
    return cases


@pytest.mark.parametrize("fmt", [FP32, FP64])
def test_bruteforce_ieee_ops(fmt):
    """~650 records per format: every combination of {+0,-0,1.5,SUB,+INF,-INF,NaN}
    through real IEEE ops; each record scanned alone so its (kind, flow) is
    checked against numpy's classification of the real result."""
    cases = _brute_records(fmt)
    rcp = OP_RCP if fmt == FP32 else OP_RCP64H
    ops_seen = set()
    for op, dest, srcs in cases:
        op = rcp if op == OP_RCP else op
        ops_seen.add(op)
        tr = Trace()
        tr.add_value_record(9, op, fmt, 0xFFFFFFFF, None if dest is None else _bits(fmt, dest),
                            [_bits(fmt, s) for s in srcs])
        hdr, arena = tr.arrays()
        exp_d, exp_f, exp_det = _ieee_expect(fmt, op, dest, srcs)
        for mode, exp in ((DEST, exp_d), (FLOW, exp_f), (FLOW_DETAIL, exp_f)):
            t = oracle.Table()
            t.scan_records(hdr, arena, mode=mode)
            ents = t.entries()
            got = None if len(ents) == 0 else (int(ents[0]["kind"]), int(ents[0]["flow"]))
            assert len(ents) <= 1
            assert got == exp, (op, dest, srcs, mode, got, exp)
            if got is not None:
                assert int(ents[0]["count"]) == 32
                assert int(ents[0]["detail"]) == (exp_det if mode == FLOW_DETAIL else 0), (op, srcs, ents)
    assert ops_seen == ({OP_FADD, OP_FMUL, OP_DIV, OP_FMNMX, OP_FSETP, OP_FSET, OP_FSEL, OP_FFMA, OP_RCP} if fmt == FP32
                        else {OP_FADD, OP_FMUL, OP_DIV, OP_FMNMX, OP_DSETP, OP_FSEL, OP_FFMA, OP_RCP64H})


# --------------------------------------------------------------------------
# aggregation: brute force over tiny random traces, pure Python + numpy
# --------------------------------------------------------------------------
def test_tiny_trace_bruteforce_dest():
    rng = np.random.default_rng(11)
    pool32 = [0x3F800000, 0x00000000, 0x80000000, 0x7F800000, 0xFF800000, 0x7FC00000, 0x00000001, 0x12345678]
    tr = Trace(seed=12)
    ref = {}
    ops = [OP_FADD, OP_FFMA, OP_RCP, OP_FSETP]
    for r in range(300):
        op = int(rng.choice(ops))
        site = int(rng.integers(0, 6))
        mask = int(rng.integers(0, 2**32)) if rng.random() < 0.3 else 0xFFFFFFFF
        vals = rng.choice(pool32, size=32)
        dest = None if op == OP_FSETP else [vals]
        tr.add(site, op, FP32, mask, [] if dest is None else dest, [])
        if dest is None:
            continue
        cls = np_class(FP32, vals.astype(np.uint64))
        for lane in range(32):
            if not (mask >> lane) & 1:
                continue
            c = int(cls[lane])
            if op == OP_RCP:
                k = DIV0 if c in (C_NAN, C_INF) else None
            else:
                k = {C_NAN: NAN, C_INF: INF, C_SUB: SUB}.get(c)
            if k is None:
                continue
            e = ref.setdefault((site, FP32, NONE, k), [0, 2**64 - 1])
            e[0] += 1
            e[1] = min(e[1], 50 + r)
    hdr, arena = tr.arrays()
    t = oracle.Table()
    t.scan_records(hdr, arena, base_index=50, mode=DEST)
    assert table_dict(t.entries()) == ref


def test_inactive_garbage_and_empty_mask():
    tr = Trace(seed=5)
    # every lane holds NaN, but only the mask decides
    tr.add(1, OP_FADD, FP32, 0x00000000, [0x7FC00000], [])
    tr.add(1, OP_FADD, FP32, 0x80000001, [0x7FC00000], [])
    hdr, arena = tr.arrays()
    t = oracle.Table()
    t.scan_records(hdr, arena)
    ents = t.entries()
    assert len(ents) == 1 and int(ents[0]["count"]) == 2 and int(ents[0]["first_index"]) == 1


def test_bad_records_counted_and_skipped():
    tr = Trace()
    tr.add(0xFFFFFFFF, OP_FADD, FP32, 0xFFFFFFFF, [0x7FC00000], [])  # invalid site
    good = tr.add(3, OP_FADD, FP32, 0xFFFFFFFF, [0x7FC00000], [])
    hdr, arena = tr.arrays()
    bad = [dict(meta=(1 << 15) | 1 | (1 << 12)),   # reserved bit
           dict(meta=25 | (1 << 12)),              # opclass out of range
           dict(meta=1 | (5 << 12)),               # dwords > 4
           dict(meta=7 | (1 << 8) | (1 << 12)),    # FP64 with odd dwords
           dict(val_off=10**6)]                    # planes outside the arena
    rows = [hdr[0], hdr[1]]
    for b in bad:
        h = hdr[1].copy()
        for k, v in b.items():
            h[k] = v
        rows.append(h)
    hdr2 = np.array(rows, dtype=hdr.dtype)
    t = oracle.Table()
    t.scan_records(hdr2, arena)
    assert t.bad_records == 6
    ents = t.entries()
    assert len(ents) == 1 and int(ents[0]["first_index"]) == good
    # FLOW mode additionally rejects packed / multi-value records (reading R13)
    tr = Trace()
    tr.add(3, 15, FP16, 0xFFFFFFFF, [0x7C007C00], [])
    h, a = tr.arrays()
    t = oracle.Table()
    t.scan_records(h, a, mode=FLOW)
    assert t.bad_records == 1 and len(t.entries()) == 0
    t = oracle.Table()
    t.scan_records(h, a, mode=DEST)
    assert t.bad_records == 0 and int(t.entries()[0]["count"]) == 64


def test_packed_and_hmma_values_per_lane():
    tr = Trace()
    # HADD2 FP16x2: low half NaN, high half SUB
    tr.add(1, 15, FP16, 0x0000000F, [0x0001_7E00], [])
    # HMMA with F32 accumulator: 4 FP32 values per lane, values 1 and 3 INF
    tr.add(2, 18, FP32, 0x00000003, [0x3F800000, 0x7F800000, 0x3F800000, 0xFF800000], [])
    # HMMA with F16 accumulator: 2 words = 4 halves per lane; one of them is +INF
    tr.add(3, 18, FP16, 0x00000001, [0x3C00_3C00, 0x7C00_3C00], [])
    hdr, arena = tr.arrays()
    t = oracle.Table()
    t.scan_records(hdr, arena)
    d = table_dict(t.entries())
    assert d == {
        (1, FP16, NONE, NAN): [4, 0], (1, FP16, NONE, SUB): [4, 0],
        (2, FP32, NONE, INF): [4, 1],
        (3, FP16, NONE, INF): [1, 2],
    }


def test_streaming_base_index_split_equals_single_scan():
    p = fpxgen.Params(seed=21, n_records=3000, n_sites=30, recipe=fpxgen.RECIPE_MIX)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 60)
    fpxgen.apply_host(w, hdr, arena)
    whole = oracle.Table()
    whole.scan_records(hdr, arena, base_index=0)
    parts = oracle.Table()
    for a, b in ((0, 1000), (1000, 1001), (1001, 3000)):
        parts.scan_records(hdr[a:b], arena, base_index=a)
    assert table_dict(whole.entries()) == table_dict(parts.entries())


# --------------------------------------------------------------------------
# synthetic traces: oracle == closed-form aggregate of the planted events
# --------------------------------------------------------------------------
@pytest.mark.parametrize(
    "recipe,flow",
    [(fpxgen.RECIPE_C1, False), (fpxgen.RECIPE_MIX, False), (fpxgen.RECIPE_FLOW, True),
     (fpxgen.RECIPE_FLOW, False), (fpxgen.RECIPE_PACKED, False)],
)
def test_planted_events_closed_form(recipe, flow):
    p = fpxgen.Params(seed=0x5EED0000 + recipe, n_records=20000, n_sites=200, recipe=recipe, p_fp64=0.5)
    hdr, arena = fpxgen.generate_host(p)
    inj, w = fpxgen.plan_injections(p, 150, flow=(recipe == fpxgen.RECIPE_FLOW))
    assert len(inj) > 100
    fpxgen.apply_host(w, hdr, arena)
    mode = FLOW if flow else DEST
    t = oracle.Table()
    t.scan_records(hdr, arena, base_index=123, mode=mode)
    assert t.bad_records == 0
    exp = expected_from_injections(hdr, inj, base_index=123, mode=mode)
    assert table_dict(t.entries()) == {k: v for k, v in exp.items()}


def test_dense_nan_stress_closed_form():
    p = fpxgen.Params(seed=7, n_records=5000, n_sites=50, recipe=fpxgen.RECIPE_STRESS, dense_nan=1.0)
    hdr, arena = fpxgen.generate_host(p)
    t = oracle.Table()
    t.scan_records(hdr, arena)
    exp = {}
    for r, h in enumerate(hdr):
        e = exp.setdefault((int(h["site"]), FP32, NONE, NAN), [0, 2**64 - 1])
        e[0] += bin(int(h["active_mask"])).count("1")
        e[1] = min(e[1], r)
    exp = {k: v for k, v in exp.items() if v[0] > 0}
    assert table_dict(t.entries()) == exp


def test_tensor_scan_vs_numpy():
    rng = np.random.default_rng(9)
    for fmt, dt in ((FP32, np.uint32), (FP64, np.uint64), (FP16, np.uint16), (BF16, np.uint16)):
        bits = rng.integers(0, np.iinfo(dt).max, 50000, dtype=dt, endpoint=True)
        t = oracle.Table()
        t.scan_tensor(bits, fmt, site=4, base_index=10)
        cls = np_class(fmt, bits.astype(np.uint64))
        exp = {}
        for c, k in ((C_NAN, NAN), (C_INF, INF), (C_SUB, SUB)):
            idx = np.nonzero(cls == c)[0]
            if len(idx):
                exp[(4, fmt, NONE, k)] = [len(idx), 10 + int(idx[0])]
        assert table_dict(t.entries()) == exp


def test_key_layout():
    assert oracle.key(0x12345678, FP64, PROP, DIV0) == (0x12345678 << 32) | (1 << 4) | (2 << 2) | 3
    assert words_of(FP64, 0x7FF0000000000001) == [1, 0x7FF00000]


# --------------------------------------------------------------------------
# R19: a recorded division on packed FP16x2 / BF16x2 words is checked per
# half, each half with the dividend / divisor halves at the same position;
# pinned against real half-precision IEEE division (numpy float16, torch
# bfloat16 on the CPU) and numpy's classification of the real quotient.
# --------------------------------------------------------------------------
_HALF_SPECIALS = {
    FP16: [0x0000, 0x8000, 0x3E00, 0x0123, 0x7C00, 0xFC00, 0x7E00],  # +0 -0 1.5 SUB +INF -INF NaN
    BF16: [0x0000, 0x8000, 0x3FC0, 0x0012, 0x7F80, 0xFF80, 0x7FC0],
}


def _half_div(fmt, a, b):
    """IEEE quotient of two halves (bit patterns) in the half format itself."""
    if fmt == FP16:
        x = np.array([a, b], np.uint16).view(np.float16)
        with np.errstate(all="ignore"):
            return int(np.array([x[0] / x[1]], np.float16).view(np.uint16)[0])
    import torch

    x = torch.tensor([a, b], dtype=torch.int32).to(torch.int16).view(torch.bfloat16)
    return int((x[0:1] / x[1:2]).view(torch.int16).to(torch.int32)[0]) & 0xFFFF


@pytest.mark.parametrize("fmt", [FP16, BF16])
def test_div_packed_halves_vs_ieee(fmt):
    sp = _HALF_SPECIALS[fmt]
    combos = list(itertools.product(sp, sp))
    tr = Trace(seed=19)
    exp = {}
    for i, (a0, b0) in enumerate(combos):
        a1, b1 = combos[(7 * i + 3) % len(combos)]
        q0, q1 = _half_div(fmt, a0, b0), _half_div(fmt, a1, b1)
        tr.add(i, OP_DIV, fmt, 0xFFFFFFFF, [q0 | (q1 << 16)], [[a0 | (a1 << 16)], [b0 | (b1 << 16)]])
        for a, b, q in ((a0, b0, q0), (a1, b1, q1)):
            fa = np_class(fmt, np.array([a], np.uint64))[0]
            a_finite_nonzero = fa in (C_SUB, CLEAN) and (a & 0x7FFF) != 0
            if (b & 0x7FFF) == 0 and a_finite_nonzero:  # IEEE divideByZero (R1)
                k = DIV0
            else:
                k = {C_NAN: NAN, C_INF: INF, C_SUB: SUB}.get(int(np_class(fmt, np.array([q], np.uint64))[0]))
            if k is not None:
                e = exp.setdefault((i, fmt, NONE, k), [0, i])
                e[0] += 32
    hdr, arena = tr.arrays()
    t = oracle.Table()
    t.scan_records(hdr, arena, mode=DEST)
    assert t.bad_records == 0
    got = table_dict(t.entries())
    assert got == exp
    assert {k[3] for k in exp} == {NAN, INF, SUB, DIV0}  # every kind occurs
    # R19: with a multi-word destination (dwords != source width) the rule
    # falls back to the destination class: 1/0 = INF reports INF, not DIV0
    tr = Trace()
    one = 0x3C00 if fmt == FP16 else 0x3F80
    inf = 0x7C00 if fmt == FP16 else 0x7F80
    tr.add(1, OP_DIV, fmt, 0x1, [inf | (one << 16), one | (one << 16)], [[one | (one << 16)], [0]])
    h, a = tr.arrays()
    t = oracle.Table()
    t.scan_records(h, a)
    assert table_dict(t.entries()) == {(1, fmt, NONE, INF): [1, 0]}


# --------------------------------------------------------------------------
# opclasses without a special rule (OTHER, MUFU_OTHER, HADD2 / HFMA2 / HMUL2,
# HMMA): the destination class of every value (Alg1's non-RCP branch, R11,
# R13), pinned per value against numpy's IEEE predicates, each format
# ----------------------------------------------------------------------------
@pytest.mark.parametrize("opclass", [0, 6, 15, 16, 17, 18])
def test_plain_class_opclasses_vs_numpy(opclass):
    rng = np.random.default_rng(opclass)
    pools = {
        FP32: [0x0, 0x80000000, 0x1, 0x7FFFFF, 0x800000, 0x7F800000, 0xFF800000, 0x7FC00000, 0x7F800001, 0x3F800000],
        FP16: [0x0, 0x8000, 0x1, 0x3FF, 0x400, 0x7C00, 0xFC00, 0x7E00, 0x7C01, 0x3C00],
        BF16: [0x0, 0x8000, 0x1, 0x7F, 0x80, 0x7F80, 0xFF80, 0x7FC0, 0x7F81, 0x3F80],
    }
    tr = Trace(seed=opclass)
    exp = {}
    for r, fmt in enumerate([FP32, FP16, BF16] * 4):
        dw = 1 + r % 4 if opclass == 18 else 1
        words = []
        vals = []
        for _ in range(dw):
            if fmt == FP32:
                v = rng.choice(pools[FP32], size=32).astype(np.uint64)
                words.append(v)
                vals.append(v)
            else:
                lo = rng.choice(pools[fmt], size=32).astype(np.uint64)
                hi = rng.choice(pools[fmt], size=32).astype(np.uint64)
                words.append(lo | (hi << np.uint64(16)))
                vals += [lo, hi]
        mask = int(rng.integers(1, 2**32))
        tr.add(r, opclass, fmt, mask, words, [])
        act = np.array([(mask >> l) & 1 for l in range(32)], dtype=bool)
        for v in vals:
            cls = np_class(fmt, v)
            for c, k in ((C_NAN, NAN), (C_INF, INF), (C_SUB, SUB)):
                cnt = int(((cls == c) & act).sum())
                if cnt:
                    e = exp.setdefault((r, fmt, NONE, k), [0, r])
                    e[0] += cnt
    hdr, arena = tr.arrays()
    t = oracle.Table()
    t.scan_records(hdr, arena)
    assert t.bad_records == 0
    assert table_dict(t.entries()) == exp
