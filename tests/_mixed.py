"""Seeded "zoo" traces for the mixed-code parity suite — inputs only.

Every active lane's word in every plane is drawn independently from a pool
of IEEE-754 bit patterns (±0, ±normal, ±min / max subnormal, ±smallest /
largest normal, ±INF, quiet and signalling NaN, all-ones, random bits), over
every opclass 0..19, every format, 0..3 sources and every legal destination
width, with full, partial, sparse and empty active masks.  So one warp-record
routinely holds several (kind, flow) codes at once — the normal case of
Alg2's leader loop over lanes with different exceptions.

Nothing here classifies a value: patterns are written from fixed tables and
random bits; the expected tables come from the oracle.  Also builds the
witness-isolation traces (one exceptional candidate per 32-record tile) for
the record scan's fast-path check.
"""
from __future__ import annotations

import numpy as np

from _records import HDR_DTYPE, meta

FP32, FP64, FP16, BF16 = 0, 1, 2, 3
DEST, FLOW, FLOW_DETAIL = 0, 1, 2

# fixed bit patterns (magnitudes; a random sign is applied to most draws)
POOL32 = np.array([0x00000000, 0x00000001, 0x007FFFFF, 0x00800000, 0x7F7FFFFF, 0x7F800000, 0x7FC00000,
                   0x7F800001, 0x7FFFFFFF, 0x3F800000, 0x00400000], dtype=np.uint64)
POOL64 = np.array([0x0000000000000000, 0x0000000000000001, 0x000FFFFFFFFFFFFF, 0x0000000100000000,
                   0x0010000000000000, 0x7FEFFFFFFFFFFFFF, 0x7FF0000000000000, 0x7FF8000000000000,
                   0x7FF0000000000001, 0x7FF0000100000000, 0x7FFFFFFFFFFFFFFF, 0x3FF0000000000000],
                  dtype=np.uint64)
POOL16 = np.array([0x0000, 0x0001, 0x03FF, 0x0400, 0x7BFF, 0x7C00, 0x7E00, 0x7C01, 0x7FFF, 0x3C00, 0x0200],
                  dtype=np.uint64)
POOLB16 = np.array([0x0000, 0x0001, 0x007F, 0x0080, 0x7F7F, 0x7F80, 0x7FC0, 0x7F81, 0x7FFF, 0x3F80, 0x0040],
                   dtype=np.uint64)
_BITS = {FP32: 32, FP64: 64, FP16: 16, BF16: 16}
_POOL = {FP32: POOL32, FP64: POOL64, FP16: POOL16, BF16: POOLB16}
_EXP = {FP32: (8, 23), FP64: (11, 52), FP16: (5, 10), BF16: (8, 7)}


def _draw(rng, fmt, shape, p_special):
    """Values of `fmt` (as uint64 bit patterns in the low bits): a share
    p_special (array broadcast to shape) from the special pool or random bits,
    the rest random normal numbers."""
    bits = _BITS[fmt]
    ebits, mbits = _EXP[fmt]
    emax = (1 << ebits) - 1
    one = np.uint64(1)
    # random normal: exponent in [1, emax - 1], random mantissa, random sign
    e = rng.integers(1, emax, size=shape, dtype=np.uint64)
    m = rng.integers(0, 1 << min(mbits, 62), size=shape, dtype=np.uint64)
    if mbits > 62:
        m = (m << np.uint64(mbits - 62)) | rng.integers(0, 1 << (mbits - 62), size=shape, dtype=np.uint64)
    v = (e << np.uint64(mbits)) | m
    u = rng.random(shape)
    special = u < p_special
    pool = _POOL[fmt]
    pick = rng.integers(0, len(pool) + 1, size=shape)
    sv = np.where(pick < len(pool), pool[np.minimum(pick, len(pool) - 1)],
                  rng.integers(0, 1 << min(bits, 63), size=shape, dtype=np.uint64) << np.uint64(bits - min(bits, 63)))
    v = np.where(special, sv, v)
    sign = rng.integers(0, 2, size=shape, dtype=np.uint64) << np.uint64(bits - 1)
    return (v | sign) & ((one << np.uint64(bits)) - one if bits < 64 else np.uint64(0xFFFFFFFFFFFFFFFF))


def _masks(rng, n):
    u = rng.random(n)
    full = np.full(n, 0xFFFFFFFF, dtype=np.uint64)
    partial = rng.integers(0, 1 << 32, size=n, dtype=np.uint64)
    sparse = (np.uint64(1) << rng.integers(0, 32, size=n, dtype=np.uint64)) | (
        np.uint64(1) << rng.integers(0, 32, size=n, dtype=np.uint64))
    return np.where(u < 0.45, full, np.where(u < 0.8, partial, np.where(u < 0.95, sparse, 0))).astype(np.uint32)


def zoo_trace(seed: int, n: int, flow: bool, n_sites: int = 13, p_bad_flow: float = 0.02,
              levels=((0.0, 0.02, 0.25, 0.9), (0.55, 0.2, 0.15, 0.1))):
    """(hdr, arena) of n zoo records.  flow=True shapes records for the
    analyzer (scalar FP32 / FP64, destination width 0 or one value) except a
    share p_bad_flow of packed records, which the FLOW modes must count as bad
    (reading R13); flow=False draws every legal DEST record shape.  `levels`:
    the per-block special-value shares and their probabilities."""
    rng = np.random.default_rng(seed)
    op = rng.integers(0, 20, size=n)
    if flow:
        fmt = np.where(rng.random(n) < 0.5, FP32, FP64)
        bad = rng.random(n) < p_bad_flow
        fmt = np.where(bad, rng.integers(2, 4, size=n), fmt)
        sw = np.where(fmt == FP64, 2, 1)
        dw = np.where(rng.random(n) < 0.8, sw, 0)
        dw = np.where(bad, 1, dw)
    else:
        fmt = rng.choice([FP32, FP64, FP16, BF16], size=n, p=[0.35, 0.25, 0.2, 0.2])
        sw = np.where(fmt == FP64, 2, 1)
        dw = np.where(fmt == FP64, 2 * rng.integers(0, 3, size=n), rng.integers(0, 5, size=n))
        # the common shape (dwords = one source width) most of the time, so DIV
        # records take the divide rule (R1 / R19)
        dw = np.where(rng.random(n) < 0.5, sw, dw)
    nsrc = rng.integers(0, 4, size=n)
    foot = dw + nsrc * sw
    off = np.concatenate([[0], np.cumsum(foot)[:-1]]).astype(np.uint64)
    total = int(foot.sum())
    # per block of 40 records: how exceptional the values are (clean stretches
    # keep whole tiles on the fast path; dense stretches mix many codes)
    blocks = (n + 39) // 40
    p_blk = rng.choice(list(levels[0]), size=blocks, p=list(levels[1]))
    p_rec = p_blk[np.arange(n) // 40]
    mask = _masks(rng, n)
    hdr = np.zeros(n, dtype=HDR_DTYPE)
    # few hot sites (equal keys meet inside tiles and warps) plus a long tail
    # of rare ones (many keys, many distinct first indices)
    hdr["site"] = np.where(rng.random(n) < 0.7, rng.integers(0, n_sites, size=n), rng.integers(0, 100_000, size=n))
    hdr["active_mask"] = mask
    hdr["meta"] = meta(op, fmt, nsrc, dw).astype(np.uint32)
    hdr["val_off"] = off
    arena = rng.integers(0, 1 << 32, size=(max(total, 1), 32), dtype=np.uint64).astype(np.uint32)  # garbage
    # fill every record's planes (active lanes; inactive lanes keep garbage)
    active = ((mask[:, None].astype(np.uint64) >> np.arange(32, dtype=np.uint64)) & 1).astype(bool)
    for f in (FP32, FP64, FP16, BF16):
        sel = np.nonzero(fmt == f)[0]
        if len(sel) == 0:
            continue
        maxw = int(foot[sel].max())
        for w in range(0, maxw, 2 if f == FP64 else 1):
            rs = sel[foot[sel] > w]
            if len(rs) == 0:
                continue
            shape = (len(rs), 32)
            p = np.broadcast_to(p_rec[rs][:, None], shape)
            if f == FP64:
                v = _draw(rng, FP64, shape, p)
                lo, hi = (v & np.uint64(0xFFFFFFFF)).astype(np.uint32), (v >> np.uint64(32)).astype(np.uint32)
                cur_lo, cur_hi = arena[off[rs] + w], arena[off[rs] + w + 1]
                arena[off[rs] + w] = np.where(active[rs], lo, cur_lo)
                arena[off[rs] + w + 1] = np.where(active[rs], hi, cur_hi)
            else:
                if f == FP32:
                    word = _draw(rng, FP32, shape, p)
                else:
                    word = _draw(rng, f, shape, p) | (_draw(rng, f, shape, p) << np.uint64(16))
                cur = arena[off[rs] + w]
                arena[off[rs] + w] = np.where(active[rs], word.astype(np.uint32), cur)
    return hdr, arena[:total] if total else np.zeros((0, 32), np.uint32)


# ---------------------------------------------------------------------------
# witness isolation: one exceptional candidate per 32-record tile
# ---------------------------------------------------------------------------
def isolated_word_trace(words: np.ndarray, opclass: int, fmt: int, filler: int, seed: int = 0,
                        lanes_partial: bool = True):
    """One-plane records (FP32 / packed halves, dwords = 1), 32 per tile: the
    first record of tile t carries words[t] in lane t % 32 and `filler` (a
    clean word) in its other active lanes; the 31 records after it are all
    filler.  Tiles of one-plane records are exactly 32 aligned records in the
    record scan, so each tile's fast-path check sees one candidate alone.
    Every other tile's carrier record has a partial mask whose inactive lanes
    hold exceptional-looking garbage (all ones)."""
    rng = np.random.default_rng(seed)
    t = len(words)
    n = 32 * t
    hdr = np.zeros(n, dtype=HDR_DTYPE)
    hdr["site"] = (np.arange(n) // 32) % 7
    hdr["meta"] = meta(opclass, fmt, 0, 1)
    hdr["val_off"] = np.arange(n)
    hdr["active_mask"] = 0xFFFFFFFF
    arena = np.full((n, 32), filler, dtype=np.uint32)
    lane = np.arange(t) % 32
    carriers = 32 * np.arange(t)
    arena[carriers, lane] = words.astype(np.uint32)
    if lanes_partial:
        part = np.nonzero(np.arange(t) % 2 == 1)[0]
        m = rng.integers(0, 1 << 32, size=len(part), dtype=np.uint64) | (np.uint64(1) << lane[part].astype(np.uint64))
        hdr["active_mask"][carriers[part]] = m.astype(np.uint32)
        inact = ~((m[:, None] >> np.arange(32, dtype=np.uint64)) & 1).astype(bool)
        rows = arena[carriers[part]]
        rows[inact] = 0xFFFFFFFF
        arena[carriers[part]] = rows
    return hdr, arena


def isolated_fp64_trace(values: np.ndarray, opclass: int = 9, filler: int = 0x3FF0000000000000):
    """Two-plane FP64 records: carrier record 80 t holds values[t] in lane
    t % 32; everything else is the clean filler.  A tile holds at most 32
    records (16 or 20 FP64 records for the 32- / 40-plane stages), so no tile
    holds two carriers whatever the ring geometry or range split."""
    t = len(values)
    per = 80
    n = per * t
    hdr = np.zeros(n, dtype=HDR_DTYPE)
    hdr["site"] = (np.arange(n) // per) % 5
    hdr["meta"] = meta(opclass, FP64, 0, 2)
    hdr["val_off"] = 2 * np.arange(n)
    hdr["active_mask"] = 0xFFFFFFFF
    arena = np.empty((2 * n, 32), dtype=np.uint32)
    arena[0::2] = filler & 0xFFFFFFFF
    arena[1::2] = filler >> 32
    lane = np.arange(t) % 32
    carriers = per * np.arange(t)
    v = values.astype(np.uint64)
    arena[2 * carriers, lane] = (v & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    arena[2 * carriers + 1, lane] = (v >> np.uint64(32)).astype(np.uint32)
    return hdr, arena


def sparse_flow_trace(seed: int, n: int):
    """Analyzer-shaped zoo records whose special values are rare (a share
    0.002 in half of the 40-record blocks): a hit tile then holds one or two
    records with an exceptional destination or source -- in any plane, FP32
    or either word of an FP64 pair, active or not -- among clean ones, the
    case the analyzer's candidate filter (exact_tile_flow) skips records in."""
    return zoo_trace(seed, n, flow=True, levels=((0.0, 0.002), (0.5, 0.5)))
