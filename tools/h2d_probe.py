"""Pinned host -> device copy bandwidth with 1..8 concurrent streams and with
64 MiB chunks: the ceiling of bench.py's e2e (19.5 GB of C2 input per step).
On the B200 boxes: 55.4-55.6 GB/s whatever the split (PCIe Gen5 x16)."""
import torch, time
n = 8 << 30  # 8 GiB
h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
d = torch.empty(n, dtype=torch.uint8, device="cuda")
for ns in (1, 2, 4, 8):
    streams = [torch.cuda.Stream() for _ in range(ns)]
    best = 0
    for rep in range(3):
        torch.cuda.synchronize()
        t = time.perf_counter()
        ch = n // ns
        for i, s in enumerate(streams):
            with torch.cuda.stream(s):
                d[i * ch:(i + 1) * ch].copy_(h[i * ch:(i + 1) * ch], non_blocking=True)
        torch.cuda.synchronize()
        best = max(best, n / (time.perf_counter() - t) / 1e9)
    print(ns, "streams", round(best, 1), "GB/s")
# chunked sequential on one stream, 64 MiB chunks
torch.cuda.synchronize(); t = time.perf_counter()
ch = 64 << 20
for i in range(0, n, ch):
    d[i:i+ch].copy_(h[i:i+ch], non_blocking=True)
torch.cuda.synchronize(); print("64MiB chunks", round(n / (time.perf_counter() - t) / 1e9, 1))
