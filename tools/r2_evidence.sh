#!/bin/bash
# One GPU session of round-2 evidence: tests, smoke, headline bench, every
# config, ncu launch list + full capture of C2, DRAM traffic per config,
# storm atomics (agg / no-agg), A/B against the round-1 library, warp spread.
#   TAG=r2e1 bash tools/r2_evidence.sh
set -u
T=${TAG:-r2ev}; O=gpurun_out/$T; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,power.limit --format=csv > $O/gpu.txt 2>&1
nproc > $O/host.txt; lscpu | grep -E "Model name|^CPU\(s\)" >> $O/host.txt
python __graft_entry__.py build > $O/build.log 2>&1 || { echo BUILD FAILED; tail -30 $O/build.log; exit 1; }
if [ "${TESTS:-1}" = 1 ]; then
  timeout 1800 python -m pytest tests -m gpu -q --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
  timeout 600 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
fi
timeout 900 python bench.py --steps ${STEPS:-200} > $O/bench_c2.json 2> $O/bench_c2.err; echo "bench c2 rc=$?"; cut -c1-300 $O/bench_c2.json
: > $O/bench_other_configs.jsonl
for c in ${CONFIGS:-c1 c3 c4a c4b c4b16 c5 s1 s2}; do
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
if [ "${NCU:-1}" = 1 ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_c2.csv \
     python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu list rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 3 -c 1 -o $O/prof_c2 \
     python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "ncu full rc=$?"
  for cfg in ${TRAFFIC_CONFIGS:-c2 c3 c4a c4b c5}; do
    timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none \
      -k regex:k_scan_ -s 4 -c 1 --csv --log-file $O/traffic_$cfg.csv \
      python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "traffic $cfg rc=$?"
  done
  TAG=$T/storm CFGS="s1 s2 c2" bash tools/storm_ncu.sh
  TAG=$T/storm_noagg CFGS="s1 s2" BENCH_ARGS="--no-warp-agg" STEPS=5 bash tools/storm_ncu.sh
fi
if [ -f build/libfpx_r1.so ] && [ "${AB:-1}" = 1 ]; then
  TAG=$T/ab_r1 LIBS="build/libfpx_r1.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c2;c3;c4a;c5;c1;s1;s2" ROUNDS=1 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
fi
timeout 600 python tools/warp_times.py c2 c3 c5 > $O/warp_times.txt 2>&1; grep -E "^c[0-9]" $O/warp_times.txt
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > $O/bench_reference.json 2> $O/bench_reference.err; echo "reference rc=$?"; cut -c1-200 $O/bench_reference.json
