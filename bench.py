#!/usr/bin/env python3
"""bench.py — GPU-FPX exception scan on B200: lane-values classified per second.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--impl fpx|reference]

A "step" is one pass of the whole hot path (decode,
classify, kind rule, warp aggregation, device table; plus the NCCL merge when
N > 1) over one batch: the configuration BASELINE.json's metric is quoted on,
configs[1] = C2 (mixed FP32/FP64 trace, 1e8 records, 1e4 sites, exception
density 1e-6, destination-only check), generated in HBM by fpxgen (inputs
20+ GB >> 126 MB L2, so no L2 flush is needed between steps).

Prints ONE JSON line (rank 0).  value = lane-values classified per second over
all ranks (active lanes x values per lane), timed with CUDA events on the
launching stream, max over ranks.  See DESIGN.md §6 for every field.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "lane-values classified/sec"
L2_BYTES = 126 << 20  # B200 L2
UNIT = "lane-values/s"

# Workloads (BASELINE.json configs); C2 is the headline.
CONFIGS = {
    "c1": dict(name="C1: tiny FP32 trace, 1e5 FFMA/FADD/MUFU.RCP records, 200 sites, planted NaN/INF/SUB/DIV0",
               recipe=0, n=100_000, sites=200, p_fp64=0.0, mode=0, n_inj=400),
    "c2": dict(name="C2: mixed FP32/FP64 trace, 1e8 records, 1e4 sites, density 1e-6, dest-only check",
               recipe=1, n=100_000_000, sites=10_000, p_fp64=0.5, mode=0, rho=1e-6),
    "c3": dict(name="C3: flow-analysis mode, FP32/FP64 70/30 records with dest + 1..3 sources, ~1e9 lane-values",
               recipe=2, n=7_800_000, sites=1_000, p_fp64=0.3, mode=1, rho=1e-6),
    "c4a": dict(name="C4a: HADD2/HFMA2/HMUL2 FP16x2/BF16x2 + HMMA records, 1e8 records, 1e3 sites, density 1e-6",
                recipe=3, n=100_000_000, sites=1_000, p_fp64=0.0, mode=0, rho=1e-6),
    "c4b": dict(name="C4b: fpx_scan_tensor over 40 GB of BF16 model activations (2e10 torch.randn values), "
                     "sparse NaN/INF at 1e-7 plus whole-row NaN bursts",
                kind="tensor", n=20_000_000_000, dtype="bf16", rho=1e-7, sites=1, mode=0, recipe=-1, p_fp64=0.0),
    "c4b16": dict(name="C4b (FP16): fpx_scan_tensor over 40 GB of FP16 torch.randn activations (2e10 values; "
                       "natural subnormals at ~4.9e-5), sparse NaN/INF at 1e-7 plus whole-row NaN bursts",
                  kind="tensor", n=20_000_000_000, dtype="fp16", rho=1e-7, sites=1, mode=0, recipe=-1, p_fp64=0.0),
    "s1": dict(name="S (stress): 1e7 FP32 FFMA records over 200 sites, every active lane NaN (rho = 1)",
               recipe=4, n=10_000_000, sites=200, p_fp64=0.0, mode=0, n_inj=0, dense=1.0),
    "s2": dict(name="S (stress): 1e7 FP32 FFMA records over 200 sites, NaN density 1e-2",
               recipe=4, n=10_000_000, sites=200, p_fp64=0.0, mode=0, n_inj=0, dense=0.01),
    "c5": dict(name="C5 shard: FP32 dest-only trace, 10^11 lane-values / 8 GPUs = 3.9e8 records per GPU, 1e6 sites",
               recipe=1, n=390_625_000, sites=1_000_000, p_fp64=0.0, mode=0, rho=1e-6),
    # at P = 1 the full C5 trace (450 GB) is scanned as
    # regenerated chunks, scan time only -- T1 of the scaling efficiency T1/(P T_P)
    "c5full": dict(name="C5 at P=1: the whole FP32 dest-only trace, 10^11 lane-values = 3.125e9 records over 1e6 "
                        "sites, scanned as 8 regenerated in-HBM chunks of 3.9e8 records (scan time only)",
                   recipe=1, n=3_125_000_000, sites=1_000_000, p_fp64=0.0, mode=0, rho=1e-6, chunks=8),
}


# The paper's headline (context, not the target: another metric on other hardware).
PAPER_CONTEXT = {
    "claim": "GPU-FPX vs BinFPE: 16x geomean end-to-end runtime speedup of NVBit-instrumented programs",
    "hardware": "RTX 2070 SUPER (Turing) + Ryzen 5 3600, or RTX 3060 (Ampere) + i9-10900K",
    "workload": "151 HPC / ML programs, FP32 + FP64 SASS",
    "cite": "PAPER.md:29 (abstract), PAPER.md:462 (machines); BASELINE.md",
    "comparable": False,
}


def config_seed(name: str) -> int:
    """The seed of a config's synthetic input (0x5EED0000 + config).
    c5full is the same trace as the c5 shards (rank r's shard = chunk r)."""
    if name == "c5full":
        name = "c5"
    return 0x5EED0000 + list(CONFIGS).index(name) + 1


def load_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class ClockSampler:
    """SM clocks / throttle reasons (NVML, else nvidia-smi) sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._t = None
        self._one = None

    def _nvml(self):
        """NVML handle and a one-sample reader (None if NVML is unavailable)."""
        try:
            import pynvml

            pynvml.nvmlInit()
            dev = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            bits = (pynvml.nvmlClocksEventReasonHwSlowdown, pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                    pynvml.nvmlClocksEventReasonSwThermalSlowdown, pynvml.nvmlClocksEventReasonSwPowerCap)
            mx = pynvml.nvmlDeviceGetMaxClockInfo(dev, pynvml.NVML_CLOCK_SM)

            def one():
                sm = pynvml.nvmlDeviceGetClockInfo(dev, pynvml.NVML_CLOCK_SM)
                r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(dev)
                self.samples.append([str(sm), str(mx), hex(r)] + ["Active" if r & b else "Not Active" for b in bits])

            one()  # fails here, before the timed region, if NVML cannot read this GPU
            return one
        except Exception:
            return None

    def _run(self):
        # NVML (what nvidia-smi reads) every 10 ms; nvidia-smi itself takes
        # ~0.3 s per query, too slow for a sub-second timed region
        if self._one is not None:
            while not self._stop.wait(0.01):
                try:
                    self._one()
                except Exception:
                    return
            return
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=5)
                if out.returncode == 0 and out.stdout.strip():
                    self.samples.append([x.strip() for x in out.stdout.strip().split(",")])
            except Exception:
                pass
            self._stop.wait(0.05)

    def __enter__(self):
        self._one = self._nvml()  # NVML set up (and one sample taken) before the timed region starts
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)
        if self._one is not None:  # and one as it ends, so short regions hold two
            try:
                self._one()
            except Exception:
                pass

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if len(s) > 3 + i and s[3 + i] == "Active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def workload_stats(hdr_dev, mode: int):
    """(lane-values per pass, algorithmic bytes per pass) from the headers on
    device: lane-values = active lanes x values per lane (DEST: destination
    values; FLOW: destination + source values); bytes = 16 B header + 128 B
    per plane the mode must read."""
    import torch

    h = hdr_dev.to(torch.int64) & 0xFFFFFFFF
    mask, meta = h[:, 1], h[:, 2]
    op, fmt, nsrc, dw = meta & 0xFF, (meta >> 8) & 3, (meta >> 10) & 3, (meta >> 12) & 7
    x = mask - ((mask >> 1) & 0x55555555)
    x = (x & 0x33333333) + ((x >> 2) & 0x33333333)
    x = (x + (x >> 4)) & 0x0F0F0F0F
    pop = (x * 0x01010101 & 0xFFFFFFFF) >> 24
    sw = torch.where(fmt == 1, 2, 1)
    nv = torch.where(fmt == 1, dw // 2, torch.where(fmt == 0, dw, 2 * dw))
    compare = (op == 11) | (op == 12) | (op == 14)
    if mode == 0:
        planes = torch.where(compare, 0, dw)
        vals = torch.where(compare, 0, nv)
    else:
        planes = dw + nsrc * sw
        vals = torch.where(dw > 0, 1, 0) + nsrc
    lane_values = int((pop * vals).sum().item())
    nbytes = 16 * h.shape[0] + 128 * int(planes.sum().item())
    return lane_values, nbytes


def build_trace(cfg, rank, world, seed):
    """This rank's shard of the configured trace, generated in HBM, with the
    planted events applied.  Weak scaling: every rank holds cfg['n'] records;
    rank r owns global records [r*n, (r+1)*n)."""
    import fpxgen

    n = cfg["n"]
    r0 = rank * n
    p = fpxgen.Params(seed=seed, n_records=n, n_sites=cfg["sites"], recipe=cfg["recipe"], p_fp64=cfg["p_fp64"],
                      dense_nan=cfg.get("dense", 0.0))
    hdr, arena, planes = fpxgen.generate_device(p, r0=r0)
    n_inj = cfg["n_inj"] if "n_inj" in cfg else int(round(cfg["rho"] * n * 32))
    inj, writes = fpxgen.plan_injections(p, n_inj, flow=cfg["mode"] == 1, r0=r0)
    fpxgen.apply_device(writes, hdr, arena)
    return p, hdr, arena, planes, r0, inj


def cpu_model() -> str:
    """The host CPU's model name (lscpu's "Model name", from /proc/cpuinfo)."""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


class PinnedToOneCore:
    """SURVEY §8(d) oracle-1c: the single-thread oracle pinned to one core
    with sched_setaffinity for the duration of the timing."""

    def __enter__(self):
        self.prev = os.sched_getaffinity(0)
        self.core = min(self.prev)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *a):
        os.sched_setaffinity(0, self.prev)


def cpu_baseline_oracle(cfg, seed, budget_s: float = 12.0):
    """The oracle (never tuned) on a bounded prefix of the same trace, single
    thread pinned to one host core of this box: lane-values/s."""
    import fpxgen
    import oracle

    def run(n):
        p = fpxgen.Params(seed=seed, n_records=n, n_sites=cfg["sites"], recipe=cfg["recipe"], p_fp64=cfg["p_fp64"])
        hdr, arena = fpxgen.generate_host(p)
        _, w = fpxgen.plan_injections(p, max(1, int(round(cfg.get("rho", 1e-6) * n * 32))), flow=cfg["mode"] == 1)
        fpxgen.apply_host(w, hdr, arena)
        t = oracle.Table()
        with PinnedToOneCore() as pin:
            t0 = time.perf_counter()
            t.scan_records(hdr, arena, base_index=0, mode=cfg["mode"])
            dt = time.perf_counter() - t0
        return t.lane_values, dt, (hdr.nbytes + arena.nbytes) / n, pin.core

    lv, dt, _, _ = run(20_000)
    n = int(min(cfg["n"], max(20_000, 20_000 * budget_s / max(dt, 1e-6))))
    lv, dt, bpr, core = run(n)
    return {"value": lv / dt, "unit": UNIT, "cores": 1, "kind": "oracle", "bytes_per_record": bpr,
            "cpu_model": cpu_model(), "pinned_core": core,
            "sample": f"first {n} records of the same {cfg['name'].split(':')[0]} trace (same seed), "
                      f"single-threaded C++ oracle pinned to core {core} (sched_setaffinity), scan only, "
                      f"{dt:.1f} s, {lv} lane-values"}


def cpu_baseline_oracle_nc(cfg, seed, single, mem_budget=12e9):
    """SURVEY §8(d) oracle-Nc: nproc processes of the unmodified oracle over
    contiguous record shards (~12 GB of trace in total), merged on the host.
    Time = slowest shard's scan + the host merge (generation excluded, as in
    the single-thread figure, which is kept as `single_core`)."""
    procs = os.cpu_count() or 1
    bpr = single["bytes_per_record"]
    per = int(max(1000, min(cfg["n"] // procs, mem_budget / procs / bpr)))
    n_inj = 0 if "n_inj" in cfg else max(1, int(round(cfg.get("rho", 1e-6) * per * 32)))
    tool = os.path.join(ROOT, "tools", "oracle_shard.py")
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    ps = [subprocess.Popen([sys.executable, tool, json.dumps(cfg), str(seed), str(i * per), str(per), str(n_inj)],
                           stdout=subprocess.PIPE, text=True, env=env) for i in range(procs)]
    res = []
    for pr in ps:
        out, _ = pr.communicate(timeout=600)
        if pr.returncode != 0:
            raise RuntimeError(f"oracle shard failed (rc {pr.returncode})")
        d = json.loads(out.strip().splitlines()[-1])
        res.append((d["lane_values"], d["seconds"], d["entries"]))
    t0 = time.perf_counter()
    merged = {}
    for _, _, ents in res:
        for site, kind, flow, fmt, detail, count, first in ents:
            k = (site, kind, flow, fmt, detail)
            c = merged.get(k)
            merged[k] = (count, first) if c is None else (c[0] + count, min(c[1], first))
    dt_merge = time.perf_counter() - t0
    lv = sum(r[0] for r in res)
    dt = max(r[1] for r in res) + dt_merge
    return {"value": lv / dt, "unit": UNIT, "cores": procs, "kind": "oracle", "cpu_model": cpu_model(),
            "sample": f"{procs} processes x {per} records (contiguous shards of the same "
                      f"{cfg['name'].split(':')[0]} trace, same seed), unmodified C++ oracle per process, slowest "
                      f"shard {max(r[1] for r in res):.2f} s + host merge {dt_merge:.3f} s, {lv} lane-values",
            "single_core": {"value": single["value"], "cores": 1, "pinned_core": single["pinned_core"],
                            "sample": single["sample"]}}


def run_reference(args, cfg, seed):
    """--impl reference: the CPU oracle as the reference arm."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import fpxgen
    import oracle

    if cfg.get("kind") == "tensor":
        return run_reference_tensor(args, cfg, seed)
    # Each step: every host core runs the unmodified oracle over its own
    # contiguous shard of the same trace (persistent worker processes,
    # tools/oracle_shard.py --serve), ~0.25 s of oracle time per shard; the
    # step time is the slowest shard plus the host merge of the shard tables.
    probe_n = 20_000
    p = fpxgen.Params(seed=seed, n_records=probe_n, n_sites=cfg["sites"], recipe=cfg["recipe"], p_fp64=cfg["p_fp64"])
    hdr, arena = fpxgen.generate_host(p)
    t = oracle.Table()
    t0 = time.perf_counter()
    t.scan_records(hdr, arena, mode=cfg["mode"])
    dt = time.perf_counter() - t0
    procs = os.cpu_count() or 1
    n = int(max(1000, min(cfg["n"] // procs, probe_n * 0.25 / max(dt, 1e-6))))
    n_inj = 0 if "n_inj" in cfg else max(1, int(round(cfg.get("rho", 1e-6) * n * 32)))
    tool = os.path.join(ROOT, "tools", "oracle_shard.py")
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    ws = [subprocess.Popen([sys.executable, tool, json.dumps(cfg), str(seed), str(i * n), str(n), str(n_inj),
                            "--serve"], stdin=subprocess.PIPE, stdout=subprocess.PIPE, text=True, env=env)
          for i in range(procs)]
    for w in ws:
        assert json.loads(w.stdout.readline()).get("ready"), "oracle shard failed to start"

    def step():
        for w in ws:
            w.stdin.write("scan\n")
            w.stdin.flush()
        res = [json.loads(w.stdout.readline()) for w in ws]
        t0 = time.perf_counter()
        merged = {}
        for r in res:
            for site, kind, flow, fmt, detail, count, first in r["entries"]:
                k = (site, kind, flow, fmt, detail)
                c = merged.get(k)
                merged[k] = (count, first) if c is None else (c[0] + count, min(c[1], first))
        return sum(r["lane_values"] for r in res), max(r["seconds"] for r in res) + time.perf_counter() - t0

    try:
        for _ in range(args.warmup):
            step()
        lv_total, dt_total = 0, 0.0
        for _ in range(args.steps):
            lv, dt = step()
            lv_total += lv
            dt_total += dt
    finally:
        for w in ws:
            try:
                w.stdin.write("quit\n")
                w.stdin.close()
            except OSError:
                pass
            w.wait(timeout=60)
    value = lv_total / dt_total
    sample = (f"{procs} processes x {n} records per step (contiguous shards of the {cfg['name'].split(':')[0]} "
              f"trace, same seed), unmodified C++ oracle per process; step = slowest shard + host merge")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt_total / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": cfg["name"], "records_per_step": n * procs, "mode": ["dest", "flow"][cfg["mode"]]},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": procs, "kind": "oracle", "cpu_model": cpu_model(),
                         "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def run_reference_tensor(args, cfg, seed):
    """--impl reference for C4b: the oracle's tensor scan on a host sample."""
    import torch

    import oracle

    g = torch.Generator().manual_seed(seed)
    n = 1 << 24
    dt = {"bf16": torch.bfloat16, "fp16": torch.float16, "fp32": torch.float32}[cfg["dtype"]]
    x = torch.randn(n, generator=g, dtype=torch.float32).to(dt)
    x[torch.randint(0, n, (max(1, int(cfg["rho"] * n)),), generator=g)] = float("nan")
    host = x.view(torch_int_view(x)).numpy()
    fmt = {"bf16": 3, "fp16": 2, "fp32": 0}[cfg["dtype"]]
    for _ in range(args.warmup):
        oracle.Table().scan_tensor(host, fmt, site=0)
    dt_total = 0.0
    for _ in range(args.steps):
        t = oracle.Table()
        t0 = time.perf_counter()
        t.scan_tensor(host, fmt, site=0)
        dt_total += time.perf_counter() - t0
    value = n * args.steps / dt_total
    sample = f"{n} {cfg['dtype'].upper()} torch.randn values per step (same recipe as C4b), single-threaded oracle"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt_total / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u16", "data": "synthetic",
        "config": {"workload": cfg["name"], "elements_per_step": n},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "cpu_model": cpu_model(),
                         "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)
    return 0


class RecordsWorkload:
    """A record trace (configs C1-C3, C4a, C5) generated in HBM by fpxgen."""

    def __init__(self, cfg, rank, seed, variant):
        self.cfg, self.seed = cfg, seed
        self.p, self.hdr, self.arena, self.planes, self.r0, self.inj = build_trace(cfg, rank, 1, seed)
        self.lane_values, self.nbytes = workload_stats(self.hdr, cfg["mode"])
        self.kernel = "k_scan_records_" + variant
        self._host = None

    def scan(self, h, stream):
        h.scan_records(self.hdr, self.arena, base_index=self.r0, mode=self.cfg["mode"], stream=stream,
                       n_records=self.cfg["n"], arena_planes=self.planes)

    def make_host_copies(self):
        import torch

        hh = torch.empty(self.hdr.shape, dtype=self.hdr.dtype, pin_memory=True)
        ah = torch.empty(self.arena.shape, dtype=self.arena.dtype, pin_memory=True)
        hh.copy_(self.hdr)
        ah.copy_(self.arena)
        self._host = (hh, ah)

    def h2d(self):
        hh, ah = self._host
        self.hdr.copy_(hh, non_blocking=True)
        self.arena.copy_(ah, non_blocking=True)
        return hh.numel() * 4 + ah.numel() * 4

    def drop_host_copies(self):
        self._host = None

    def config(self):
        return {"records_per_gpu": self.cfg["n"], "sites": self.cfg["sites"],
                "mode": ["dest", "flow"][self.cfg["mode"]], "planted_events": int(len(self.inj))}

    def cpu_baseline(self):
        single = cpu_baseline_oracle(self.cfg, self.seed)
        if (os.cpu_count() or 1) == 1:
            single.pop("bytes_per_record")
            return single
        return cpu_baseline_oracle_nc(self.cfg, self.seed, single)


class ChunkedRecordsWorkload:
    """c5full: a trace larger than HBM (450 GB) scanned as regenerated chunks
    (SURVEY §8(d) "at P = 1 ... scanned as regenerated chunks").  Chunk c holds
    global records [c*m, (c+1)*m) (the c5 shard of rank c), generated in HBM
    and planted, then scanned with base_index = c*m; only the scans are timed
    (CUDA events around each chunk's scan), the regeneration is not."""

    chunked = True

    def __init__(self, cfg, rank, seed, variant):
        self.cfg, self.seed = cfg, seed
        self.chunks = cfg["chunks"]
        self.m = cfg["n"] // self.chunks
        assert self.m * self.chunks == cfg["n"]
        self.kernel = "k_scan_records_" + variant
        self.lane_values, self.nbytes, self.planted = 0, 0, 0
        self.scan_ms = []  # per chunk scan, last step
        self._buf = None
        # workload statistics of every chunk (one generation pass)
        for c in range(self.chunks):
            self._make(c)
            lv, nb = workload_stats(self._buf[0], cfg["mode"])
            self.lane_values += lv
            self.nbytes += nb
            self.planted += len(self._inj)
        self._cur = self.chunks - 1

    def _make(self, c):
        import fpxgen

        cfg = self.cfg
        p = fpxgen.Params(seed=self.seed, n_records=self.m, n_sites=cfg["sites"], recipe=cfg["recipe"],
                          p_fp64=cfg["p_fp64"])
        self._buf = None  # free the previous chunk first (two would not fit at once)
        hdr, arena, planes = fpxgen.generate_device(p, r0=c * self.m)
        inj, writes = fpxgen.plan_injections(p, int(round(cfg["rho"] * self.m * 32)), r0=c * self.m)
        fpxgen.apply_device(writes, hdr, arena)
        self._buf, self._inj, self._planes, self._cur = (hdr, arena), inj, planes, c

    def scan(self, h, stream):
        """One step = every chunk: regenerate (untimed), scan (timed)."""
        import torch

        self.scan_ms = []
        order = [self._cur] + [c for c in range(self.chunks) if c != self._cur]  # reuse the resident chunk first
        evs = []
        for c in order:
            if c != self._cur:
                torch.cuda.synchronize()
                self._make(c)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            hdr, arena = self._buf
            h.scan_records(hdr, arena, base_index=c * self.m, mode=self.cfg["mode"], stream=stream, n_records=self.m,
                           arena_planes=self._planes)
            b.record(stream)
            evs.append((a, b))
            torch.cuda.synchronize()  # the next regeneration overwrites this chunk
        self.scan_ms = [a.elapsed_time(b) for a, b in evs]

    def config(self):
        return {"records_total": self.cfg["n"], "chunks": self.chunks, "records_per_chunk": self.m,
                "sites": self.cfg["sites"], "mode": "dest", "planted_events": int(self.planted),
                "timed": "sum of the chunk scans (regeneration of each chunk in HBM is outside the timed region)"}

    def make_host_copies(self):
        raise NotImplementedError("c5full (450 GB) has no host copy: e2e is measured on c5")

    def cpu_baseline(self):
        single = cpu_baseline_oracle(self.cfg, self.seed)
        if (os.cpu_count() or 1) == 1:
            single.pop("bytes_per_record")
            return single
        return cpu_baseline_oracle_nc(self.cfg, self.seed, single)


class TensorWorkload:
    """C4b: a plain activation buffer (torch.randn, seeded) with planted NaN/INF."""

    def __init__(self, cfg, rank, seed, dev):
        import torch

        self.cfg, self.seed = cfg, seed
        n = cfg["n"]
        dt = {"bf16": torch.bfloat16, "fp16": torch.float16, "fp32": torch.float32}[cfg["dtype"]]
        g = torch.Generator(device=dev).manual_seed(seed + rank)
        self.x = torch.empty(n, dtype=dt, device=dev)
        chunk = 1 << 30
        for a in range(0, n, chunk):  # randn in chunks keeps the fp32 temporaries small
            b = min(n, a + chunk)
            self.x[a:b] = torch.randn(b - a, generator=g, device=dev, dtype=torch.float32).to(dt)
        n_inj = int(round(cfg["rho"] * n))
        idx = torch.randint(0, n, (n_inj,), generator=g, device=dev)
        self.x[idx[: n_inj // 2]] = float("nan")
        self.x[idx[n_inj // 2:]] = float("inf")
        for r in range(4):  # SRU-style uninitialised rows: whole 4096-value rows of NaN
            row = int(torch.randint(0, n // 4096, (1,), generator=g, device=dev)) * 4096
            self.x[row: row + 4096] = float("nan")
        self.base = rank * n
        self.lane_values = n
        self.nbytes = n * self.x.element_size()
        self.kernel = "k_scan_tensor"
        self.planted = n_inj + 4 * 4096
        self._host = None

    def scan(self, h, stream):
        h.scan_tensor(self.x, site=0, base_index=self.base, stream=stream)

    def make_host_copies(self):
        import torch

        self._host = torch.empty(self.x.shape, dtype=self.x.dtype, pin_memory=True)
        self._host.copy_(self.x)

    def h2d(self):
        self.x.copy_(self._host, non_blocking=True)
        return self._host.numel() * self._host.element_size()

    def drop_host_copies(self):
        self._host = None

    def config(self):
        return {"elements_per_gpu": self.cfg["n"], "dtype": self.cfg["dtype"], "planted_events": self.planted}

    def cpu_baseline(self, budget_s: float = 12.0):
        import oracle

        fmt = {"bf16": 3, "fp16": 2, "fp32": 0}[self.cfg["dtype"]]
        m = 1 << 24
        host = self.x[:m].view(torch_int_view(self.x)).cpu().numpy()
        t = oracle.Table()
        t0 = time.perf_counter()
        t.scan_tensor(host, fmt, site=0)
        dt = time.perf_counter() - t0
        m2 = int(min(self.cfg["n"], m * budget_s / max(dt, 1e-6)))
        host = self.x[:m2].view(torch_int_view(self.x)).cpu().numpy()
        t = oracle.Table()
        t0 = time.perf_counter()
        t.scan_tensor(host, fmt, site=0)
        dt = time.perf_counter() - t0
        return {"value": m2 / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
                "sample": f"first {m2} elements of the same C4b buffer, single-threaded C++ oracle, {dt:.1f} s"}


def torch_int_view(x):
    import torch

    return {2: torch.int16, 4: torch.int32, 8: torch.int64}[x.element_size()]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="c2", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="fpx", choices=["fpx", "reference"])
    ap.add_argument("--records", type=int, default=0, help="override the record count (debug only)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--variant", default="tma", choices=["tma", "ldg"], help="record-scan kernel (ldg = ablation)")
    ap.add_argument("--no-warp-agg", action="store_true",
                    help="ablation: per-lane table updates in the exact path (FPX_OPT_NO_WARP_AGG)")
    ap.add_argument("--debug-one-gpu", action="store_true",
                    help="testing only: every rank on cuda:0 with gloo (exercises the N > 1 code paths on one GPU)")
    ap.add_argument("--merge", default="nccl", choices=["nccl", "peer"],
                    help="N > 1: NCCL merge of per-GPU tables (default; SURVEY §8 e), or one shared table updated "
                         "over NVLink peer memory with system-scope atomics (not yet run across distinct GPUs)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    cfg = dict(CONFIGS[args.config])
    if args.records:
        cfg["n"] = args.records - args.records % cfg.get("chunks", 1)
    seed = config_seed(args.config)

    if args.impl == "reference":
        return run_reference(args, cfg, seed)

    import torch
    import torch.distributed as dist

    from paper_conf_hpdc_lilfslg23_b200 import dist as fdist
    from paper_conf_hpdc_lilfslg23_b200 import fpx

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    assert world == args.gpus or world == 1, "launch N>1 with torchrun"
    if args.debug_one_gpu:
        local = 0
    torch.cuda.set_device(local)
    if world > 1 and args.debug_one_gpu:
        dist.init_process_group("gloo")
    elif world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)

    hflags = (fpx.OPT_SCAN_LDG if args.variant == "ldg" else 0) | (fpx.OPT_NO_WARP_AGG if args.no_warp_agg else 0)
    h = fpx.Handle(local, flags=hflags)
    stream = torch.cuda.current_stream(dev)
    if cfg.get("kind") == "tensor":
        wl = TensorWorkload(cfg, rank, seed, dev)
    elif cfg.get("chunks"):
        wl = ChunkedRecordsWorkload(cfg, rank, seed, args.variant)
    else:
        wl = RecordsWorkload(cfg, rank, seed, args.variant)
    chunked = getattr(wl, "chunked", False)
    torch.cuda.synchronize()

    shared, merge_note = None, None
    if world > 1 and args.merge == "peer":
        try:
            shared = fdist.SharedTable(local, flags=hflags)
            h.close()
            h = shared.handle
        except RuntimeError as ex:  # no peer / IPC access: fall back to the NCCL merge, and say so
            merge_note = f"peer table unavailable ({str(ex)[:120]}); NCCL merge used"
    merged = [None]

    def step(ev_a=None, ev_b=None):
        if shared is not None:
            shared.reset(stream=stream)  # home clears; everyone waits
        else:
            h.reset(stream=stream)
        if ev_a is not None:
            ev_a.record(stream)
        wl.scan(h, stream)
        if ev_b is not None:
            ev_b.record(stream)
        if shared is not None:
            shared.finish(stream=stream)  # every rank's inserts landed in the home table
        elif world > 1:
            merged[0] = fdist.merge_handle(h, stream=stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    K = args.steps
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    # Inputs that fit the 126 MB L2 (C1) would be re-read from L2 by every
    # step: write a 2 x L2 buffer between steps instead, outside per-step
    # events that then make up the timed total.
    flush = None
    if wl.nbytes < 2 * L2_BYTES:
        flush = torch.zeros(2 * L2_BYTES // 4, dtype=torch.int32, device=dev)
        sevs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    bounds = [torch.cuda.Event(enable_timing=True) for _ in range(K + 1)]
    chunk_ms = []  # chunked workload: per step, the scan time of every chunk
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t_start.record(stream)
        for i in range(K):
            if flush is not None:
                flush.add_(1)
                sevs[i][0].record(stream)
            bounds[i].record(stream)
            step(*evs[i])
            if flush is not None:
                sevs[i][1].record(stream)
            if chunked:
                chunk_ms.append(list(wl.scan_ms))
        bounds[K].record(stream)
        t_end.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    if chunked:  # scan time only: the chunks' regeneration is not part of a step
        step_ms = [sum(c) for c in chunk_ms]
        kern_ms = float(np.mean([x for c in chunk_ms for x in c]))
    else:
        step_ms = ([a.elapsed_time(b) for a, b in sevs] if flush is not None else
                   [bounds[i].elapsed_time(bounds[i + 1]) for i in range(K)])
        kern_ms = float(np.mean([a.elapsed_time(b) for a, b in evs]))
    total_ms = t_start.elapsed_time(t_end) if (flush is None and not chunked) else sum(step_ms)
    median_ms = float(np.median(step_ms))
    per_rank = None
    lane_values, nbytes = wl.lane_values, wl.nbytes
    if world > 1:
        # max over ranks for the times; the work is summed over ranks (each
        # rank scans its own shard)
        tdev = torch.device("cpu") if dist.get_backend() == "gloo" else dev
        t = torch.zeros(world, 5, dtype=torch.float64, device=tdev)
        t[rank, 0], t[rank, 1], t[rank, 2], t[rank, 3], t[rank, 4] = total_ms, kern_ms, median_ms, lane_values, nbytes
        dist.all_reduce(t, op=dist.ReduceOp.SUM)  # each rank fills its own row
        per_rank = {"step_ms": [round(float(v) / K, 4) for v in t[:, 0]],
                    "scan_kernel_ms": [round(float(v), 4) for v in t[:, 1]]}
        total_ms, kern_ms, median_ms = float(t[:, 0].max()), float(t[:, 1].max()), float(t[:, 2].max())
        lane_values, nbytes = int(t[:, 3].sum()), int(t[:, 4].sum())
    ms_per_step = total_ms / K

    if shared is None or rank == 0:
        ents = h.fetch()
        ok_status = h.last_status
    else:
        ents, ok_status = [], 0
    if merged[0] is not None:  # NCCL merge: report the merged (global) table
        ents = merged[0][0]

    # e2e: the same metric through the public API with host buffers: per step,
    # H2D of the step's inputs from pinned memory, scan, fetch (D2H of entries).
    # N > 1: every rank copies and scans its own shard, the step ends with the
    # merged table on rank 0 in host memory (shared table: rank 0's fetch;
    # NCCL merge: the merged arrays copied to the host); time = max over ranks.
    e2e = None
    if chunked:
        e2e = {"value": None, "unit": UNIT, "note": "a 450 GB trace has no host copy to stream in; e2e is on c5"}
    elif not args.no_e2e:
        try:
            wl.make_host_copies()
            torch.cuda.synchronize()
            d2h = 0
            e_a, e_b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            tot = 0.0
            for i in range(args.e2e_steps + 1):
                torch.cuda.synchronize()
                if world > 1:
                    dist.barrier()
                e_a.record(stream)
                h2d = wl.h2d()
                if shared is not None:
                    shared.reset(stream=stream)
                else:
                    h.reset(stream=stream)
                wl.scan(h, stream)
                if shared is not None:
                    shared.finish(stream=stream)
                    got_bytes = h.fetch().nbytes if rank == 0 else 0  # synchronises; D2H of the entries
                elif world > 1:
                    k, c, f = fdist.merge_handle(h, stream=stream)
                    got_bytes = sum(t.cpu().numel() * 8 for t in (k, c, f)) if rank == 0 else 0
                else:
                    got_bytes = h.fetch().nbytes
                e_b.record(stream)
                torch.cuda.synchronize()
                if i > 0:  # first pass = warm-up
                    tot += e_a.elapsed_time(e_b)
                d2h = got_bytes
            if world > 1:
                tdev = torch.device("cpu") if dist.get_backend() == "gloo" else dev
                t = torch.tensor([tot, float(h2d), float(d2h)], dtype=torch.float64, device=tdev)
                tmax = t[:1].clone()
                dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
                dist.all_reduce(t, op=dist.ReduceOp.SUM)
                tot, h2d, d2h = float(tmax[0]), int(t[1]), int(t[2])
            e2e = {"value": lane_values / (tot / args.e2e_steps / 1e3), "unit": UNIT,
                   "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h), "steps": args.e2e_steps}
            wl.drop_host_copies()
        except Exception as ex:  # pragma: no cover - reported, not hidden
            e2e = {"value": None, "unit": UNIT, "error": str(ex)[:200]}

    if rank != 0:
        if shared is not None:
            shared.close()
        if world > 1:
            dist.destroy_process_group()
        return 0

    peak, peak_src = load_peak()
    # per GPU: one launch's algorithmic bytes (the average shard; a chunk for
    # the chunked workload) / the launch time (max over ranks)
    launches_per_step = getattr(wl, "chunks", 1)
    achieved = nbytes / world / launches_per_step / (kern_ms / 1e3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            tj = json.load(f)
        traffic = tj.get(args.config, {}).get("dram_bytes_per_launch")
    clocks = clk.summary()
    cpu = None if (args.no_cpu_baseline or world > 1) else wl.cpu_baseline()  # rank 0 at N = 1 only
    line = {
        "metric": METRIC,
        "value": lane_values / (ms_per_step / 1e3),
        "unit": UNIT,
        "n_gpus": world,
        "steps": K,
        "warmup": args.warmup,
        "ms_per_step": ms_per_step,
        "ms_per_step_median": median_ms,
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "u32",
        "data": "synthetic (fpxgen counter-based trace generated in HBM, planted exceptions)",
        "config": {
            "workload": cfg["name"],
            **wl.config(),
            "lane_values_per_step": lane_values,
            "algorithmic_bytes_per_step": nbytes,
            "work_summed_over_ranks": world > 1,
            "table_entries": int(len(ents)),
            "fetch_status": int(ok_status),
            "l2": ("inputs >> 126 MB L2 (no flush needed)" if flush is None else
                   f"inputs ({nbytes / 1e6:.0f} MB) fit the 126 MB L2: a {2 * L2_BYTES >> 20} MiB buffer is written "
                   "between timed steps, outside the per-step events that make up ms_per_step"),
            "parallelism": f"shards x{world}" + ("" if world == 1 else (" + shared table over NVLink peer memory"
                                                                         if shared is not None else
                                                                         " + NCCL merge per step")),
            **({"merge_note": merge_note} if merge_note else {}),
            **({"ablation": "variant=" + args.variant} if args.variant != "tma" else {}),
            **({"ablation_agg": "no warp aggregation (FPX_OPT_NO_WARP_AGG)"} if args.no_warp_agg else {}),
        },
        "roofline": {
            "bound": "hbm",
            "achieved": achieved,
            "peak": peak,
            "unit": "GB/s",
            "frac": achieved / peak,
            "traffic": traffic,
            "kernel": wl.kernel,
            "kernel_ms": kern_ms,
            "peak_source": peak_src,
        },
        "clocks": clocks,
        # per step: table reset (2 kernels) + scan (1); merge (N > 1): compact, iota,
        # radix sort, gather, sort, select-init, select, lookup (counted with ncu,
        # tools/count_merge_launches.py); NCCL's own kernels are not ours
        "gpu_launches": K * (2 + launches_per_step + (8 if (world > 1 and shared is None) else 0)),
        "cpu_baseline": cpu,
        "e2e": e2e,
        **({"per_rank": per_rank} if per_rank else {}),
        "paper_context": PAPER_CONTEXT,
    }
    print(json.dumps(line), flush=True)
    if shared is not None:
        shared.close()
    else:
        h.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
