"""One shard of the multi-core oracle (bench.py cpu_baseline and the
--impl reference arm): generate records [r0, r0 + n) of a synthetic trace on
the host, plant that shard's events, time the unmodified CPU oracle over it,
print one JSON line.  Runs as its own process (no torch, no CUDA).

    python tools/oracle_shard.py '<cfg json>' SEED R0 N N_INJ [--serve]

--serve: generate once, print {"ready": true}, then scan once per "scan" line
read from stdin (a fresh table each time) until "quit" or EOF.
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import fpxgen  # noqa: E402
import oracle  # noqa: E402


def main():
    cfg = json.loads(sys.argv[1])
    seed, r0, n, n_inj = (int(v) for v in sys.argv[2:6])
    p = fpxgen.Params(seed=seed, n_records=n, n_sites=cfg["sites"], recipe=cfg["recipe"], p_fp64=cfg["p_fp64"],
                      dense_nan=cfg.get("dense", 0.0))
    hdr, arena = fpxgen.generate_host(p, r0=r0)
    if n_inj:
        _, w = fpxgen.plan_injections(p, n_inj, flow=cfg["mode"] == 1, r0=r0)
        fpxgen.apply_host(w, hdr, arena)

    def scan():
        t = oracle.Table()
        t0 = time.perf_counter()
        t.scan_records(hdr, arena, base_index=r0, mode=cfg["mode"])
        dt = time.perf_counter() - t0
        ents = [[int(e[f]) for f in ("site", "kind", "flow", "fmt", "detail", "count", "first_index")]
                for e in t.entries()]
        print(json.dumps({"lane_values": int(t.lane_values), "seconds": dt, "entries": ents}), flush=True)

    if "--serve" not in sys.argv:
        scan()
        return
    print(json.dumps({"ready": True}), flush=True)
    for line in sys.stdin:
        if line.strip() != "scan":
            break
        scan()


if __name__ == "__main__":
    main()
