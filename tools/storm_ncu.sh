#!/bin/bash
# Storm-regime evidence (SURVEY §8(d) stress row): for each config, bench lines
# and one ncu capture of the record-scan launch with the L2 atomic counters,
# shared-memory atomics, divergence and issue metrics; plus a --set full
# capture of S1 for the source page.  Outputs under gpurun_out/$TAG.
#   TAG=storm CFGS="s1 s2 c2" FULL=s1 bash tools/storm_ncu.sh
set -u
OUT=gpurun_out/${TAG:-storm}; mkdir -p $OUT
python __graft_entry__.py build > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
M=gpu__time_duration.sum,lts__t_requests_srcunit_tex_op_atom.sum,lts__t_requests_srcunit_tex_op_red.sum,lts__t_sectors_op_atom.sum,lts__d_atomic_input_cycles_active.sum,lts__d_atomic_input_cycles_active.avg.pct_of_peak_sustained_elapsed,smsp__sass_inst_executed_op_global_atom.sum,smsp__sass_inst_executed_op_global_red.sum,smsp__sass_inst_executed_op_shared_atom.sum,smsp__inst_executed.sum,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__issue_active.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum
for cfg in ${CFGS:-s1 s2}; do
  for agg in ${AGGS:-""}; do :; done
  timeout 600 python bench.py --config $cfg --steps ${STEPS:-50} --warmup 3 --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} > $OUT/bench_$cfg.json 2> $OUT/bench_$cfg.err
  python -c "import json; d=json.loads(open('$OUT/bench_$cfg.json').read()); print('$cfg', round(d['roofline']['achieved']), 'GB/s', round(d['roofline']['kernel_ms'],4), 'ms', d['clocks']['sm_mhz'])"
  timeout 600 ncu --metrics $M --clock-control none -k regex:k_scan_records -s 4 -c 1 --csv --log-file $OUT/ncu_$cfg.csv \
    python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} > $OUT/ncu_$cfg.log 2>&1
  echo "ncu $cfg rc=$?"
done
for cfg in ${FULL:-}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $OUT/full_$cfg \
    python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > $OUT/full_$cfg.log 2>&1; echo "full $cfg rc=$?"
done
