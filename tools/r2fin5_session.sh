#!/bin/bash
# Last check of round 2 (final build: one-plane ring): GPU suite, smoke,
# headline bench, storm bench lines + atomics.
set -u
T=r2fin5; O=gpurun_out/$T; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { echo BUILD FAILED; tail -30 $O/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
timeout 600 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; echo "bench c2 rc=$?"; cut -c1-200 $O/bench_c2.json
TAG=$T/storm CFGS="s1 s2 c2" bash tools/storm_ncu.sh
for c in c5 c4a c3; do timeout 600 python bench.py --config $c --steps 100 --warmup 3 --no-e2e --no-cpu-baseline >> $O/bench_other_configs.jsonl 2>> $O/bench_other.err; done
timeout 900 python bench.py --config c5full --steps 3 --warmup 3 --no-cpu-baseline >> $O/bench_other_configs.jsonl 2>> $O/bench_other.err
python - $O/bench_other_configs.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); r=d['roofline']
        print(d['config']['workload'][:28], f"{d['value']:.3e} lv/s", round(r['achieved']), 'GB/s', round(r['frac'],3), round(r['kernel_ms'],4), 'ms', d['clocks']['sm_mhz'], d['clocks']['reasons'])
PY
