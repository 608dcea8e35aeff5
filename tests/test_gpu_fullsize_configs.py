"""Parity at every BASELINE.json config's full size, built and launched exactly
as bench.py times it (bench.RecordsWorkload / bench.TensorWorkload: same
seeds, same generator parameters, same kernel, one CTA per SM).

* Record configs C3 (FLOW, ~1e9 lane-values), C4a (1e8 packed / HMMA
  records) and the C5 shard (3.9e8 FP32 records, 1e6 sites): the whole GPU
  table must equal the closed-form aggregate of the planted events (derived
  from the injection list and the paper's dispatch, independent of both the
  oracle and the kernels), and 16 random windows of 2048 records (plus the
  first and the last) must match the CPU oracle entry by entry.
* C4b (40 GB of BF16 torch.randn activations with planted NaN / INF and
  whole NaN rows): per-kind counts and first indices against the IEEE
  definition evaluated by torch on the same buffer, chunk by chunk (a property
  at any size), plus 4 windows of 1e6 elements against the CPU oracle.

C2 at full size and the FP16 C4b variant are in test_gpu_fullsize.py.
"""
import numpy as np
import pytest

import fpxgen
import oracle
from _records import describe_diff, entries_equal, expected_from_injections, table_dict

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _bench():
    import importlib
    import os
    import sys

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    if root not in sys.path:
        sys.path.insert(0, root)
    return importlib.import_module("bench")


def _footprint(meta):
    """Planes a record occupies in the arena: dwords + nsrc * sw (include/fpx.h)."""
    fmt, nsrc, dw = (meta >> 8) & 3, (meta >> 10) & 3, (meta >> 12) & 7
    return dw + nsrc * np.where(fmt == 1, 2, 1)


@pytest.mark.parametrize("name", ["c3", "c4a", "c5"])
def test_record_config_full_size(name):
    from paper_conf_hpdc_lilfslg23_b200 import fpx

    bench = _bench()
    cfg = dict(bench.CONFIGS[name])
    wl = bench.RecordsWorkload(cfg, 0, bench.config_seed(name), "tma")
    mode = cfg["mode"]
    stream = torch.cuda.current_stream()
    with fpx.Handle(0) as h:
        wl.scan(h, stream)
        got = h.fetch()
        assert h.last_status == fpx.OK
    hdr_host = wl.hdr.cpu().numpy().view(fpxgen.HDR_DTYPE).reshape(-1)
    exp = expected_from_injections(hdr_host, wl.inj, wl.r0, mode)
    td = table_dict(got)
    assert td == exp, sorted((k, td.get(k), exp.get(k)) for k in set(td) ^ set(exp) | {
        k for k in td if k in exp and td[k] != exp[k]})[:8]
    assert len(exp) > 100

    n = cfg["n"]
    W = 2048
    rng = np.random.default_rng(7)
    starts = [0, n - W] + [int(v) for v in rng.integers(0, n - W, 16)]
    with fpx.Handle(0) as h:
        for w in starts:
            hw = hdr_host[w: w + W].copy()
            lo = int(hw["val_off"].min())
            hi = int((hw["val_off"].astype(np.int64) + _footprint(hw["meta"].astype(np.int64))).max())
            aw = wl.arena[lo * 32: hi * 32].cpu().numpy().view(np.uint32).reshape(-1, 32)
            hw["val_off"] -= lo
            ref = oracle.Table()
            ref.scan_records(hw, aw, base_index=wl.r0 + w, mode=mode)
            assert ref.bad_records == 0
            h.reset()
            d_h = torch.from_numpy(hw.view(np.int32).reshape(-1, 4)).cuda()
            d_a = torch.from_numpy(aw.view(np.int32).reshape(-1)).cuda()
            h.scan_records(d_h, d_a, base_index=wl.r0 + w, mode=mode)
            got = h.fetch()
            assert entries_equal(got, ref.entries()), describe_diff(got, ref.entries())
    del wl
    torch.cuda.empty_cache()


def test_c4b_bf16_full_size():
    from paper_conf_hpdc_lilfslg23_b200 import fpx

    bench = _bench()
    cfg = dict(bench.CONFIGS["c4b"])
    dev = torch.device("cuda", 0)
    wl = bench.TensorWorkload(cfg, 0, bench.config_seed("c4b"), dev)
    x = wl.x
    n = x.numel()
    with fpx.Handle(0) as h:
        wl.scan(h, torch.cuda.current_stream())
        got = h.fetch()
        assert h.last_status == fpx.OK

    # IEEE definition (torch's own isnan / isinf; subnormal = 0 < |x| < finfo.tiny), chunked
    tiny = torch.finfo(torch.bfloat16).tiny
    acc = {}
    chunk = 1 << 30
    for a in range(0, n, chunk):
        xs = x[a: a + chunk]
        for kind, m in ((fpx.NAN, torch.isnan(xs)), (fpx.INF, torch.isinf(xs)),
                        (fpx.SUB, (xs.abs() < tiny) & (xs != 0))):
            cnt = int(m.sum())
            if cnt:
                c = acc.setdefault(kind, [0, None])
                c[0] += cnt
                if c[1] is None:
                    c[1] = wl.base + a + int(torch.nonzero(m)[0, 0])
            del m
    exp = {(0, fpx.BF16, 0, k): v for k, v in acc.items()}
    assert table_dict(got) == exp
    assert exp[(0, fpx.BF16, 0, fpx.NAN)][0] >= 4 * 4096

    rng = np.random.default_rng(11)
    W = 1_000_003
    starts = [0, n - W] + [int(v) for v in rng.integers(0, n - W, 2)]
    with fpx.Handle(0) as h:
        for a in starts:
            w = x[a: a + W]
            ref = oracle.Table()
            ref.scan_tensor(w.cpu().view(torch.int16).numpy().view(np.uint16), fmt=fpx.BF16, site=0,
                            base_index=wl.base + a)
            h.reset()
            h.scan_tensor(w, site=0, base_index=wl.base + a)
            got = h.fetch()
            assert entries_equal(got, ref.entries()), describe_diff(got, ref.entries())
    del wl, x
    torch.cuda.empty_cache()
