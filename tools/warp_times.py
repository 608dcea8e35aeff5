"""Load imbalance of the record scan: per-warp start / end times (%globaltimer)
of one launch, from a diagnostics build of libfpx.so (-DFPX_WARP_TIMES).

    python tools/warp_times.py [config ...]      # default: c2 c3 c4a c5

Builds build/libfpx_wt.so, scans each bench config (same trace as bench.py)
a few times and prints, for the last launch: the kernel span (last end - first
start), the warp durations (min / median / max) and the end-time spread — the
share of the span the SMs spend idle waiting for the slowest warp."""
import ctypes
import os
import subprocess
import sys

# One config per process: the per-warp arrays are device globals indexed by
# scan warp, and kernels with different scan-warp counts (the analyzer's drain
# warp) would otherwise read another config's stale entries.
_CFGS = sys.argv[1:] or ["c2", "c3", "c4a", "c5"]
if len(_CFGS) > 1:
    for _c in _CFGS:
        sys.stdout.flush()
        subprocess.run([sys.executable, os.path.abspath(__file__), _c], check=False)
    sys.exit(0)

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
# WT_SRC: build the diagnostics library from another source tree (A/B against
# an older commit's worktree); WT_TAG names the library
SRC_ROOT = os.environ.get("WT_SRC", ROOT)
LIB = os.path.join(ROOT, "build", f"libfpx_wt{os.environ.get('WT_TAG', '')}.so")
CSRC = os.path.join(SRC_ROOT, "paper_conf_hpdc_lilfslg23_b200", "csrc")
SRC = [os.path.join(CSRC, f) for f in ("fpx_api.cu", "fpx_scan_records.cu", "fpx_scan_tensor.cu", "fpx_table.cu")]

os.makedirs(os.path.dirname(LIB), exist_ok=True)
subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17", "-Xcompiler",
                "-fPIC,-O3", "-shared", "-I" + os.path.join(SRC_ROOT, "include"), "-DFPX_WARP_TIMES", *SRC, "-o", LIB],
               check=True)
os.environ["FPX_LIB"] = LIB

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_lilfslg23_b200 import fpx  # noqa: E402

wt = ctypes.CDLL(LIB)
wt.fpx_debug_warp_times.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]
NW = 148 * 32

for name in _CFGS:
    cfg = dict(bench.CONFIGS[name])
    wl = bench.RecordsWorkload(cfg, 0, bench.config_seed(name), "tma")
    stream = torch.cuda.current_stream()
    h = fpx.Handle(0)
    t0 = np.zeros(NW, dtype=np.uint64)
    t1 = np.zeros(NW, dtype=np.uint64)
    spans = []
    for rep in range(6):
        h.reset(stream=stream)
        wl.scan(h, stream)
        torch.cuda.synchronize()
        n = wt.fpx_debug_warp_times(t0.ctypes.data, t1.ctypes.data, NW)
        live = (t0[:n] != 0) & (t1[:n] >= t0[:n])
        a, b = t0[:n][live].astype(np.int64), t1[:n][live].astype(np.int64)
        hx = np.zeros(NW, dtype=np.uint64)
        ex = np.zeros(NW, dtype=np.uint64)
        if hasattr(wt, "fpx_debug_warp_exact"):
            wt.fpx_debug_warp_exact(hx.ctypes.data, ex.ctypes.data, NW)
        cnt3 = np.zeros((3, NW), dtype=np.uint64)
        if hasattr(wt, "fpx_debug_warp_counts"):
            wt.fpx_debug_warp_counts(cnt3[0].ctypes.data, cnt3[1].ctypes.data, cnt3[2].ctypes.data, NW)
        ph = np.zeros(3 * NW, dtype=np.uint64)
        if hasattr(wt, "fpx_debug_warp_phases"):
            wt.fpx_debug_warp_phases(ph.ctypes.data, NW)
        if rep >= 2:
            spans.append((a, b))
            last_exact = (hx[:n][live].astype(np.int64), ex[:n][live].astype(np.int64),
                          ph.reshape(NW, 3)[:n][live].astype(np.int64), cnt3[:, :n][:, live].astype(np.int64),
                          np.nonzero(live)[0])
        t0[:] = 0
        t1[:] = 0
    for a, b in spans[-2:]:
        s0 = a.min()
        span = b.max() - s0
        dur = b - a
        ends = np.sort(b - s0)
        idle = 1.0 - dur.sum() / (len(dur) * span)
        print(f"{name}: warps {len(dur)} span {span / 1e3:.1f} us | warp dur min/med/max "
              f"{dur.min() / 1e3:.1f}/{np.median(dur) / 1e3:.1f}/{dur.max() / 1e3:.1f} us | start spread "
              f"{(a.max() - s0) / 1e3:.1f} us | end p10/p50/p90/max {ends[len(ends) // 10] / 1e3:.1f}/"
              f"{ends[len(ends) // 2] / 1e3:.1f}/{ends[9 * len(ends) // 10] / 1e3:.1f}/{ends[-1] / 1e3:.1f} us | "
              f"idle share {100 * idle:.1f} %", flush=True)
    hits, ens, phs, c3, gws = last_exact
    if c3.sum():
        order = np.argsort(b - a)
        med = order[len(order) // 2]
        for tag, i in [("median", med)] + [("slow", i) for i in order[-6:]]:
            print(f"  {tag:6s} warp {gws[i]:5d} (CTA {gws[i] // 20:3d}) dur {(b[i] - a[i]) / 1e3:6.1f} us start "
                  f"{(a[i] - a.min()) / 1e3:5.1f} tiles {c3[0, i]:5d} chunks {c3[1, i]:3d} mbar wait "
                  f"{c3[2, i] / 1e3:6.1f} us hits {hits[i]}", flush=True)
    if phs.sum():
        late = np.argsort(b - a)[-5:]
        print("  FLOW exact phases (prologue / records / flush) of the 5 slowest warps: "
              + ", ".join(f"{phs[i, 0] / 1e3:.1f}/{phs[i, 1] / 1e3:.1f}/{phs[i, 2] / 1e3:.1f} us" for i in late), flush=True)
    if hits.sum():
        late = np.argsort(b - a)[-5:]
        print(f"  exact path: hit tiles total {hits.sum()}, per warp med/max {np.median(hits):.0f}/{hits.max()}, "
              f"time per warp med/max {np.median(ens) / 1e3:.1f}/{ens.max() / 1e3:.1f} us; 5 slowest warps: "
              + ", ".join(f"dur {(b[i] - a[i]) / 1e3:.1f} us hits {hits[i]} exact {ens[i] / 1e3:.1f} us" for i in late),
              flush=True)
    h.close()
    del wl
    torch.cuda.empty_cache()
