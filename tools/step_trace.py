"""Diagnostic: per-launch duration of the record scan over many back-to-back
steps, and with idle gaps between steps, to separate kernel speed from the
power-capped clock of a sustained run.  Not a bench line.

    python tools/step_trace.py [--config c2] [--steps 200] [--gap-ms 0,50]
"""
import argparse
import os
import subprocess
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def smi():
    q = "clocks.sm,clocks.mem,power.draw,temperature.gpu,clocks_throttle_reasons.active"
    return subprocess.run(["nvidia-smi", f"--query-gpu={q}", "--format=csv,noheader"],
                          capture_output=True, text=True).stdout.strip()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c2")
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--gap-ms", default="0,50")
    ap.add_argument("--probe", default="records", help="records | tensor (fpx_scan_tensor over as many bytes)")
    args = ap.parse_args()
    import torch

    from paper_conf_hpdc_lilfslg23_b200 import fpx

    cfg = dict(bench.CONFIGS[args.config])
    wl = bench.RecordsWorkload(cfg, 0, 1234, "tma")
    h = fpx.Handle(0)
    if args.probe == "tensor":  # same byte count, streamed by the tensor kernel
        nbytes = wl.nbytes
        del wl
        torch.cuda.empty_cache()
        x = torch.zeros(nbytes // 4, dtype=torch.float32, device="cuda")

        class W:
            pass
        wl = W()
        wl.nbytes = x.numel() * 4
        wl.scan = lambda h, s: h.scan_tensor(x, site=1, stream=s)
    elif args.probe == "copy":  # torch copy_ moving as many bytes (read + write)
        nbytes = wl.nbytes
        del wl
        torch.cuda.empty_cache()
        a = torch.zeros(nbytes // 8, dtype=torch.float32, device="cuda")
        b = torch.empty_like(a)

        class W:
            pass
        wl = W()
        wl.nbytes = a.numel() * 8
        wl.scan = lambda h, s: b.copy_(a)
    s = torch.cuda.current_stream()
    for gap in [float(g) for g in args.gap_ms.split(",")]:
        for _ in range(5):
            h.reset(stream=s)
            wl.scan(h, s)
        torch.cuda.synchronize()
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        clocks = []
        for i, (a, b) in enumerate(evs):
            h.reset(stream=s)
            a.record(s)
            wl.scan(h, s)
            b.record(s)
            if gap > 0:
                torch.cuda.synchronize()
                time.sleep(gap / 1e3)
            if i % max(args.steps // 5, 1) == 0:
                clocks.append(smi())
        torch.cuda.synchronize()
        ms = [a.elapsed_time(b) for a, b in evs]
        gbs = [wl.nbytes / (m / 1e3) / 1e9 for m in ms]
        q = sorted(gbs)
        print(f"gap {gap} ms: first5 {[round(g) for g in gbs[:5]]} last5 {[round(g) for g in gbs[-5:]]} "
              f"median {q[len(q) // 2]:.0f} max {q[-1]:.0f} min {q[0]:.0f} GB/s")
        for c in clocks:
            print("   smi:", c)


if __name__ == "__main__":
    main()
