#!/bin/bash
# Final evidence of round 2 session 2 (after the BF16 list merge and the
# CTA-table reductions): GPU suite, smoke, headline bench, every config,
# ncu launch list + full capture of C2, DRAM traffic of C2 / C4a, storm atomics.
set -u
T=r2fin2; O=gpurun_out/$T; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,power.limit --format=csv > $O/gpu.txt 2>&1
python __graft_entry__.py build > $O/build.log 2>&1 || { echo BUILD FAILED; tail -30 $O/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
timeout 600 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; echo "bench c2 rc=$?"; cut -c1-300 $O/bench_c2.json
: > $O/bench_other_configs.jsonl
for c in c1 c3 c4a c4b c4b16 c5 s1 s2; do
  timeout 600 python bench.py --config $c --steps 100 --warmup 3 --no-e2e --no-cpu-baseline >> $O/bench_other_configs.jsonl 2>> $O/bench_other.err
done
timeout 900 python bench.py --config c5full --steps 3 --warmup 3 --no-cpu-baseline >> $O/bench_other_configs.jsonl 2>> $O/bench_other.err
python - $O/bench_other_configs.jsonl <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); r=d['roofline']
        print(d['config']['workload'][:28], f"{d['value']:.3e} lv/s", round(r['achieved']), 'GB/s', round(r['frac'],3), round(r['kernel_ms'],4), 'ms', d['clocks']['sm_mhz'], d['clocks']['reasons'])
PY
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_c2.csv \
   python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 3 -c 1 -o $O/prof_c2 \
   python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu full rc=$?"
for cfg in c2 c4a; do
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none \
    -k regex:k_scan_ -s 4 -c 1 --csv --log-file $O/traffic_$cfg.csv \
    python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "traffic $cfg rc=$?"
done
TAG=$T/storm CFGS="s1 s2 c2" bash tools/storm_ncu.sh
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > $O/bench_reference.json 2> $O/bench_reference.err; echo "reference rc=$?"
