"""Early notification (§3.1.2: new exceptions reach the host "before
(hour-long) GPU runs finish"): fpx_poll_new reports a planted key while the
scans that find it are still in flight, without synchronising any stream,
and the final table is unchanged by the option."""
import time

import numpy as np
import pytest

import fpxgen
import oracle
from _mixed import sparse_flow_trace
from _records import DEST, FP32, NAN, NONE, OP_FADD, Trace, describe_diff, entries_equal, table_dict

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
DEV = "cuda:0"


@pytest.fixture(scope="module")
def fpx():
    from paper_conf_hpdc_lilfslg23_b200 import fpx as m

    return m


def test_poll_sees_planted_key_before_the_scans_finish(fpx):
    # a clean 2e7-record FP32 trace (~2.9 GB) scanned 40 times back to back
    # (~0.4 s of device work); one early record holds one NaN lane
    p = fpxgen.Params(seed=5, n_records=20_000_000, n_sites=1000, recipe=fpxgen.RECIPE_MIX, p_fp64=0.0)
    hdr, arena, planes = fpxgen.generate_device(p)
    head = hdr[:100].cpu().numpy().view(np.uint32).reshape(-1, 4)
    # an early FADD / FMUL / FFMA record (one FP32 destination word) with lane 17 active
    r = next(i for i in range(100) if (head[i, 2] & 0xFF) in (1, 2, 3) and (head[i, 1] >> 17) & 1)
    site = int(head[r, 0])
    arena[int(head[r, 3]) * 32 + 17] = 0x7FC00001  # lane 17 of its destination word: NaN
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    with fpx.Handle(0, flags=fpx.OPT_LIVE_NEW) as h:
        assert len(h.poll_new()) == 0
        done = []
        for i in range(40):
            h.scan_records(hdr, arena, base_index=0, stream=s, n_records=p.n_records, arena_planes=planes)
            ev = torch.cuda.Event()
            ev.record(s)
            done.append(ev)
        seen, t0 = [], time.perf_counter()
        while not len(seen) and time.perf_counter() - t0 < 30:
            seen = h.poll_new()
        finished = sum(e.query() for e in done)
        busy = not s.query()
        assert len(seen) == 1
        e = seen[0]
        assert (int(e["site"]), int(e["fmt"]), int(e["flow"]), int(e["kind"])) == (site, FP32, NONE, NAN)
        assert int(e["first_index"]) == r and int(e["count"]) == 1  # the inserting event
        assert busy and finished < 40, (finished, busy)  # reported while scans were still running
        s.synchronize()
        assert len(h.poll_new()) == 0  # each key once
        assert table_dict(h.fetch()) == {(site, FP32, NONE, NAN): [40, r]}
        h.reset()
        assert len(h.poll_new()) == 0  # a reset restarts the ring; the old key is not re-reported
        h.scan_records(hdr, arena, base_index=10, n_records=p.n_records, arena_planes=planes)
        torch.cuda.synchronize()
        again = h.poll_new()
        assert len(again) == 1 and int(again[0]["first_index"]) == 10 + r


@pytest.mark.parametrize("storm", [False, True], ids=["sparse", "storm"])
def test_live_option_same_table_and_every_new_key_once(fpx, storm):
    """With FPX_OPT_LIVE_NEW the fetched table equals the oracle's and every
    key is polled exactly once across batches (poll keys == FETCH_ALL keys);
    also through the storm kernel, which inserts a CTA's new keys when the
    CTA finishes."""
    p = fpxgen.Params(seed=9, n_records=300_000, n_sites=5000, recipe=fpxgen.RECIPE_MIX)
    hdr, arena = fpxgen.generate_host(p)
    _, w = fpxgen.plan_injections(p, 3000)
    fpxgen.apply_host(w, hdr, arena)
    d_hdr = torch.from_numpy(hdr.view(np.int32).reshape(-1, 4)).to(DEV)
    d_arena = torch.from_numpy(arena.view(np.int32).reshape(-1)).to(DEV)
    ref = oracle.Table()
    ref.scan_records(hdr, arena, base_index=0)
    with fpx.Handle(0, flags=fpx.OPT_LIVE_NEW | (fpx.OPT_STORM if storm else 0)) as h:
        polled = []
        for a, b in ((0, 100_000), (100_000, 300_000)):
            h.scan_records(d_hdr[a:b], d_arena, base_index=a, arena_planes=arena.shape[0])
            torch.cuda.synchronize()
            polled.append(h.poll_new(capacity=1 << 16))
        got = h.fetch()
    assert entries_equal(got, ref.entries()), describe_diff(got, ref.entries())
    keys = lambda es: sorted((int(e["site"]), int(e["fmt"]), int(e["flow"]), int(e["kind"])) for e in es)
    allp = np.concatenate(polled)
    assert keys(allp) == keys(got) and len(set(keys(allp))) == len(allp)
    final = table_dict(got)
    for e in allp:  # provisional values are bounded by the final ones
        c, f = final[(int(e["site"]), int(e["fmt"]), int(e["flow"]), int(e["kind"]))]
        assert 1 <= int(e["count"]) <= c and int(e["first_index"]) >= f


@pytest.mark.parametrize("mode", [1, 2], ids=["flow", "flow_detail"])
def test_analyzer_live_and_fetch_new(fpx, mode):
    """The analyzer kernels hand their table updates to the CTA's drain warp
    (EventQueue): the table, the live ring and the FETCH_NEW windows must be
    exactly what the scanning warps' own inserts gave -- every key once in the
    ring and once across the FETCH_NEW windows, the table equal to the
    oracle's."""
    hdr, arena = sparse_flow_trace(seed=23, n=400_000)
    d_hdr = torch.from_numpy(hdr.view(np.int32).reshape(-1, 4)).to(DEV)
    d_arena = torch.from_numpy(arena.view(np.int32).reshape(-1)).to(DEV)
    ref = oracle.Table()
    ref.scan_records(hdr, arena, base_index=0, mode=mode)
    with fpx.Handle(0, flags=fpx.OPT_LIVE_NEW) as h:
        polled, windows = [], []
        for a, b in ((0, 150_000), (150_000, 400_000)):
            h.scan_records(d_hdr[a:b], d_arena, base_index=a, mode=mode, arena_planes=arena.shape[0])
            torch.cuda.synchronize()
            polled.append(h.poll_new(capacity=1 << 16))
            windows.append(h.fetch_new())
        got = h.fetch()
    assert entries_equal(got, ref.entries()), describe_diff(got, ref.entries())
    keys = lambda es: sorted((int(e["site"]), int(e["fmt"]), int(e["flow"]), int(e["kind"]), int(e["detail"]))
                             for e in es)
    allp, alln = np.concatenate(polled), np.concatenate(windows)
    assert keys(allp) == keys(got) and len(set(keys(allp))) == len(allp)
    assert keys(alln) == keys(got) and len(set(keys(alln))) == len(alln)
    assert {int(e["flow"]) for e in got} == {1, 2, 3}


def test_poll_without_option_is_invalid(fpx):
    with fpx.Handle(0) as h:
        with pytest.raises(fpx.FpxError):
            h.poll_new()
