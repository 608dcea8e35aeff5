#!/bin/bash
# One GPU session: build, parity tests, a short bench, the ncu launch list and
# one full ncu capture of the record-scan kernel.  Outputs under gpurun_out/.
set -u
OUT=gpurun_out/${TAG:-run}
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,power.limit --format=csv > $OUT/gpu.txt 2>&1
nproc > $OUT/host.txt; lscpu | grep -E "Model name|^CPU\(s\)" >> $OUT/host.txt
python __graft_entry__.py build > $OUT/build.log 2>&1 || { echo BUILD FAILED; tail -50 $OUT/build.log; exit 1; }
if [ "${TESTS:-1}" = 1 ]; then
  timeout 900 python -m pytest tests -m gpu -x -q --timeout 240 ${PYTEST_ARGS:-} > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
  tail -30 $OUT/pytest_gpu.log
fi
if [ "${BENCH:-1}" = 1 ]; then
  timeout 900 python bench.py ${BENCH_ARGS:-} > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; cat $OUT/bench.json; tail -5 $OUT/bench.err
fi
if [ "${NCU:-1}" = 1 ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches.csv \
     python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline ${NCU_BENCH_ARGS:-} > $OUT/ncu_launch_bench.log 2>&1; echo "ncu list rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 3 -c 1 -o $OUT/prof_records \
     python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline ${NCU_FULL_ARGS:-} > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
  tail -3 $OUT/ncu_full.log
fi
if [ -n "${EXTRA:-}" ]; then
  i=0
  IFS=';' read -ra CMDS <<< "$EXTRA"
  for c in "${CMDS[@]}"; do
    i=$((i+1)); echo "== extra $i: $c" >> $OUT/extra.log
    timeout 600 bash -c "$c" >> $OUT/extra.log 2>&1; echo "rc=$?" >> $OUT/extra.log
  done
  grep -E '^==|^\{|rc=' $OUT/extra.log | cut -c1-400
fi
if [ "${NCU_TENSOR:-0}" = 1 ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_tensor -s 3 -c 1 -o $OUT/prof_tensor \
     python bench.py --config c4b --records 1000000000 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/ncu_tensor.log 2>&1; echo "ncu tensor rc=$?"
fi
if [ "${NCU_TRAFFIC:-0}" = 1 ]; then
  # DRAM bytes of the dominant kernel at the full bench configuration (1 replay pass)
  for cfg in ${TRAFFIC_CONFIGS:-c2}; do
    timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
      -k regex:k_scan_ -s 4 -c 1 --csv --log-file $OUT/traffic_$cfg.csv \
      python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > $OUT/traffic_$cfg.log 2>&1; echo "traffic $cfg rc=$?"
  done
fi
if [ "${SMOKE:-0}" = 1 ]; then
  timeout 600 python __graft_entry__.py smoke > $OUT/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 $OUT/smoke.log
fi
