"""CPU side of the mixed-code suite: the zoo traces and the witness-isolation
traces are what they claim to be (checked on the oracle side, no GPU).

* zoo traces hold many records whose active lanes carry two or more distinct
  (kind, flow) codes, every opclass 0..19 and every format;
* the isolation traces' oracle tables equal the closed form computed with
  numpy's IEEE predicates (another pin of the oracle's classification over
  every exceptional FP16 / BF16 half in both word positions and the FP32 /
  FP64 boundary sets, through the record path).
"""
import numpy as np
import pytest

import oracle
from _mixed import isolated_fp64_trace, isolated_word_trace, zoo_trace
from _records import BF16, DEST, FLOW, FP16, FP32, FP64, NONE, np_class, table_dict

KIND = {1: 0, 2: 1, 3: 2}


def test_zoo_mixes_codes_within_records():
    hdr, arena = zoo_trace(seed=7, n=4000, flow=False)
    assert set(int(m) & 0xFF for m in hdr["meta"]) == set(range(20))
    assert set((int(m) >> 8) & 3 for m in hdr["meta"]) == {0, 1, 2, 3}
    multi = 0
    for r in range(len(hdr)):
        t = oracle.Table()
        t.scan_records(hdr[r:r + 1], arena, mode=DEST)
        multi += len(t) >= 2
    assert multi > 300
    hdr, arena = zoo_trace(seed=8, n=4000, flow=True)
    multi = 0
    for r in range(len(hdr)):
        t = oracle.Table()
        t.scan_records(hdr[r:r + 1], arena, mode=FLOW)
        multi += len(t) >= 2
    assert multi > 300


def _closed(fmt, values, sites, first_of):
    cls = np_class(fmt, values.astype(np.uint64))
    exp = {}
    for t, c in enumerate(cls):
        if c:
            e = exp.setdefault((int(sites[t]), fmt, NONE, KIND[int(c)]), [0, first_of(t)])
            e[0] += 1
    return exp


@pytest.mark.parametrize("fmt", [FP16, BF16])
def test_isolation_trace_closed_form_halves(fmt):
    allv = np.arange(65536, dtype=np.uint64)
    exc = allv[np_class(fmt, allv) != 0]
    one = 0x3C00 if fmt == FP16 else 0x3F80
    words = np.concatenate([exc | np.uint64(0x8000 << 16), (exc << np.uint64(16)) | np.uint64(0x8000),
                            exc | np.uint64(one << 16)])
    halves = np.concatenate([exc, exc, exc])
    hdr, arena = isolated_word_trace(words, opclass=15, fmt=fmt, filler=one | (one << 16))
    t = oracle.Table()
    t.scan_records(hdr, arena)
    assert table_dict(t.entries()) == _closed(fmt, halves, np.arange(len(words)) % 7, lambda i: 32 * i)


def test_isolation_trace_closed_form_fp64():
    his = [0x00000000, 0x00000001, 0x000FFFFF, 0x00100000, 0x7FEFFFFF, 0x7FF00000, 0x7FF00001, 0x7FFFFFFF]
    v = np.array([(h << 32) | l for h in his for l in (0, 1, 0x80000000)], dtype=np.uint64)
    hdr, arena = isolated_fp64_trace(v)
    t = oracle.Table()
    t.scan_records(hdr, arena)
    assert table_dict(t.entries()) == _closed(FP64, v, np.arange(len(v)) % 5, lambda i: 80 * i)
    w = np.array([1, 0x7FFFFF, 0x800000, 0x7F800000, 0x7F800001, 0x80000001], dtype=np.uint64)
    hdr, arena = isolated_word_trace(w, opclass=1, fmt=FP32, filler=0x3F800000)
    t = oracle.Table()
    t.scan_records(hdr, arena)
    assert table_dict(t.entries()) == _closed(FP32, w, np.arange(len(w)) % 7, lambda i: 32 * i)
