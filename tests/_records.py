"""Test helpers: build hand-made record traces and independent expectations.

Nothing here imports the oracle or the product; the helpers only lay out
input bytes in the record format of include/fpx.h and compute expectations
with numpy's own IEEE routines (np.isnan / np.isinf / finfo.tiny), which is
independent of the oracle's bit-field classification.
"""
from __future__ import annotations

import json
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
HDR_DTYPE = np.dtype([("site", "<u4"), ("active_mask", "<u4"), ("meta", "<u4"), ("val_off", "<u4")])
ENTRY_FIELDS = ("site", "kind", "flow", "fmt", "detail", "count", "first_index")

FP32, FP64, FP16, BF16 = 0, 1, 2, 3
NAN, INF, SUB, DIV0 = 0, 1, 2, 3
NONE, GEN, PROP, KILL = 0, 1, 2, 3
DEST, FLOW, FLOW_DETAIL = 0, 1, 2
OP_FADD, OP_FMUL, OP_FFMA, OP_RCP, OP_RCP64H, OP_MUFU = 1, 2, 3, 4, 5, 6
OP_DADD, OP_DMUL, OP_DFMA, OP_FSEL, OP_FSET, OP_FSETP, OP_FMNMX, OP_DSETP = 7, 8, 9, 10, 11, 12, 13, 14
OP_HADD2, OP_HFMA2, OP_HMUL2, OP_HMMA, OP_DIV = 15, 16, 17, 18, 19


def meta(opclass, fmt, nsrc, dwords):
    return opclass | (fmt << 8) | (nsrc << 10) | (dwords << 12)


def sw(fmt):
    return 2 if fmt == FP64 else 1


def words_of(fmt, bits):
    """32-bit words of one value for a register plane: FP64 -> (lo, hi)."""
    if fmt == FP64:
        return [bits & 0xFFFFFFFF, bits >> 32]
    return [bits & 0xFFFFFFFF]


class Trace:
    """Append records one by one; lanes not in the mask get garbage words."""

    def __init__(self, seed=0):
        self.hdr = []
        self.planes = []
        self.rng = np.random.default_rng(seed)

    def add(self, site, opclass, fmt, mask, dest_words, src_words, dwords=None):
        """dest_words: list over planes of per-lane arrays (len 32) or scalars;
        src_words: list over sources of lists over planes (sw planes each)."""
        nsrc = len(src_words)
        if dwords is None:
            dwords = len(dest_words)
        off = len(self.planes)
        garbage = lambda: self.rng.integers(0, 2**32, size=32, dtype=np.uint64).astype(np.uint32)
        for w in list(dest_words) + [p for s in src_words for p in s]:
            plane = garbage()
            vals = np.broadcast_to(np.asarray(w, dtype=np.uint64).astype(np.uint32), (32,))
            m = np.array([(mask >> l) & 1 for l in range(32)], dtype=bool)
            plane[m] = vals[m]
            self.planes.append(plane)
        self.hdr.append((site, mask, meta(opclass, fmt, nsrc, dwords), off))
        return len(self.hdr) - 1

    def add_value_record(self, site, opclass, fmt, mask, dest_bits, src_bits):
        """Scalar record with one destination value (or None) and source values."""
        dest = [] if dest_bits is None else words_of(fmt, dest_bits)
        srcs = [words_of(fmt, s) for s in src_bits]
        return self.add(site, opclass, fmt, mask, dest, srcs)

    def arrays(self):
        hdr = np.array(self.hdr, dtype=HDR_DTYPE)
        arena = np.array(self.planes, dtype=np.uint32).reshape(-1, 32) if self.planes else np.zeros((0, 32), np.uint32)
        return hdr, arena


def load_worked_cases():
    with open(os.path.join(HERE, "golden", "worked_cases.json")) as f:
        return json.load(f)["cases"]


# ---- independent classification with numpy's IEEE routines ----------------
def np_class(fmt, bits):
    """0 clean, 1 NaN, 2 INF, 3 SUB via numpy float predicates (not bit fields)."""
    bits = np.asarray(bits, dtype=np.uint64)
    if fmt == FP32:
        x = bits.astype(np.uint32).view(np.float32)
        tiny = np.finfo(np.float32).tiny
    elif fmt == FP64:
        x = bits.view(np.float64)
        tiny = np.finfo(np.float64).tiny
    elif fmt == FP16:
        x = bits.astype(np.uint16).view(np.float16)
        tiny = np.finfo(np.float16).tiny
    else:  # BF16: the top half of an FP32 with the same exponent field width
        x = (bits.astype(np.uint32) << np.uint32(16)).view(np.float32)
        tiny = np.finfo(np.float32).tiny
    with np.errstate(invalid="ignore"):
        out = np.zeros(x.shape, dtype=np.int64)
        out[np.isnan(x)] = 1
        out[np.isinf(x)] = 2
        out[(~np.isnan(x)) & (~np.isinf(x)) & (x != 0) & (np.abs(x) < tiny)] = 3
    return out


def entries_equal(got, exp):
    if len(got) != len(exp):
        return False
    return all(np.array_equal(np.asarray(got[f]), np.asarray(exp[f])) for f in ENTRY_FIELDS)


def describe_diff(got, exp, limit=8):
    def k(e):
        return (int(e["site"]), int(e["fmt"]), int(e["flow"]), int(e["kind"]), int(e["detail"]))

    g = {k(e): (int(e["count"]), int(e["first_index"])) for e in got}
    x = {k(e): (int(e["count"]), int(e["first_index"])) for e in exp}
    out = []
    for kk in sorted(set(g) | set(x)):
        if g.get(kk) != x.get(kk):
            out.append(f"key(site,fmt,flow,kind,detail)={kk}: got {g.get(kk)} expected {x.get(kk)}")
            if len(out) >= limit:
                break
    return f"{len(got)} vs {len(exp)} entries; " + "; ".join(out)


def expected_from_injections(hdr, inj, base_index=0, mode=DEST):
    """Closed-form table of a clean synthetic trace plus planted events
    (fpxgen): each planted lane contributes one lane-value.  Kinds follow the
    paper's dispatch: RCP destinations report DIV0; flows follow
    Table 2.  Returns a dict key -> [count, first]."""
    exp = {}
    RCP = (OP_RCP, OP_RCP64H)
    kind_of_class = {0: NAN, 1: INF, 2: SUB}
    for e in inj:
        r = int(e["record"])
        h = hdr[r]
        m = int(h["meta"])
        op, fmt = m & 0xFF, (m >> 8) & 3
        lanes = bin(int(e["lanemask"]) & int(h["active_mask"])).count("1")
        if lanes == 0:
            continue
        dc, sc = int(e["dest_class"]), int(e["src_class"])
        D = None if dc == 0xFF else (DIV0 if op in RCP else kind_of_class[dc])
        S = None if sc == 0xFF else kind_of_class[sc]
        if mode == DEST:
            if D is None:
                continue
            key = (int(h["site"]), fmt, NONE, D)
        else:
            if D is not None and S is None:
                key = (int(h["site"]), fmt, GEN, D)
            elif D is not None:
                key = (int(h["site"]), fmt, PROP, D)
            elif S is not None:
                key = (int(h["site"]), fmt, KILL, S)
            else:
                continue
        c = exp.setdefault(key, [0, 2**64 - 1])
        c[0] += lanes
        c[1] = min(c[1], base_index + r)
    return exp


def table_dict(entries):
    return {
        (int(e["site"]), int(e["fmt"]), int(e["flow"]), int(e["kind"])): [int(e["count"]), int(e["first_index"])]
        for e in entries
    }
