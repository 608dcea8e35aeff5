"""bench.py's JSON contract: the reference arm on CPU, the product arm and the
multi-rank path (two ranks sharing cuda:0 over gloo) on the GPU."""
import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
             "vs_baseline", "dtype", "data", "config"}


def run(args, env=None, timeout=600):
    e = dict(os.environ, **(env or {}))
    p = subprocess.run([sys.executable, *args], cwd=ROOT, capture_output=True, text=True, timeout=timeout, env=e)
    assert p.returncode == 0, p.stderr[-3000:]
    return [json.loads(line) for line in p.stdout.splitlines() if line.startswith("{")]


def free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_reference_arm_json_line():
    lines = run(["bench.py", "--impl", "reference", "--config", "c1", "--steps", "3", "--warmup", "3"],
                env={"CUDA_VISIBLE_DEVICES": ""})
    assert len(lines) == 1
    d = lines[0]
    assert BASE_KEYS <= set(d) and d["impl"] == "reference"
    assert d["metric"] == "lane-values classified/sec" and d["value"] > 0 and d["steps"] == 3
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


def test_reference_arm_nonzero_rank_is_silent():
    lines = run(["bench.py", "--impl", "reference", "--config", "c1", "--steps", "3", "--warmup", "3"],
                env={"CUDA_VISIBLE_DEVICES": "", "RANK": "1", "WORLD_SIZE": "2"})
    assert lines == []


@pytest.mark.gpu
def test_product_arm_json_line():
    lines = run(["bench.py", "--config", "c1", "--steps", "5", "--warmup", "3"])
    assert len(lines) == 1
    d = lines[0]
    assert BASE_KEYS <= set(d) and d["n_gpus"] == 1 and d["scaling"] == "weak"
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-9
    assert d["gpu_launches"] == 5 * 3
    assert d["ms_per_step_median"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["cpu_baseline"]["cpu_model"] and "pinned_core" in d["cpu_baseline"].get("single_core", d["cpu_baseline"])
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert {"sm_mhz", "sm_max_mhz", "reasons"} <= set(d["clocks"])
    assert d["config"]["fetch_status"] == 0 and d["config"]["table_entries"] > 0


@pytest.mark.gpu
@pytest.mark.parametrize("merge", ["nccl", "peer"])
def test_two_ranks_on_one_gpu(merge):
    """The N > 1 path (shards, merge, max-over-ranks timing, per-rank times)
    with both ranks on cuda:0 (gloo; the peer table degenerates to a same-device
    IPC mapping or falls back to the merge, saying so)."""
    lines = run(["-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2", "--master-addr=127.0.0.1",
                 f"--master-port={free_port()}", "bench.py", "--gpus", "2", "--debug-one-gpu", "--config", "c1",
                 "--steps", "3", "--warmup", "3", "--merge", merge])
    assert len(lines) == 1
    d = lines[0]
    assert d["n_gpus"] == 2 and len(d["per_rank"]["step_ms"]) == 2 and len(d["per_rank"]["scan_kernel_ms"]) == 2
    assert d["ms_per_step"] == pytest.approx(max(d["per_rank"]["step_ms"]), rel=1e-3)
    assert d["config"]["fetch_status"] == 0 and d["config"]["table_entries"] > 0
    assert d["cpu_baseline"] is None
    # e2e at N = 2: both shards copied from host memory, merged table read back on rank 0
    assert d["e2e"]["value"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["config"]["work_summed_over_ranks"] is True
    assert d["e2e"]["h2d_bytes_per_step"] >= d["config"]["algorithmic_bytes_per_step"]


@pytest.mark.gpu
def test_chunked_full_trace_json_line():
    """c5full (the whole C5 trace at P = 1, regenerated chunk by chunk; scan
    time only) at a reduced size: 8 chunks, one scan launch per chunk."""
    lines = run(["bench.py", "--config", "c5full", "--records", "8000000", "--steps", "3", "--warmup", "3",
                 "--no-cpu-baseline"])
    d = lines[0]
    assert d["config"]["chunks"] == 8 and d["config"]["records_per_chunk"] == 1_000_000
    assert d["gpu_launches"] == 3 * (2 + 8)
    assert d["e2e"]["value"] is None and d["value"] > 0
    assert d["config"]["table_entries"] > 0 and d["config"]["fetch_status"] == 0
