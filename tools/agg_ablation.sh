#!/bin/bash
# Warp-aggregation ablation (SURVEY §8(d) stress row): bench lines and L2
# atomic / reduction request counts of the record scan with and without
# FPX_OPT_NO_WARP_AGG on the NaN storms S1 (every lane NaN) and S2 (1 %).
OUT=${1:-gpurun_out/agg}; mkdir -p $OUT
M=gpu__time_duration.sum,lts__t_requests_op_atom.sum,lts__t_requests_op_red.sum,smsp__sass_inst_executed_op_global_atom.sum,smsp__sass_inst_executed_op_global_red.sum
for cfg in s1 s2 c2; do
  for agg in "" "--no-warp-agg"; do
    tag=${cfg}${agg:+_noagg}
    timeout 600 python bench.py --config $cfg --steps 30 --warmup 3 --no-e2e --no-cpu-baseline $agg > $OUT/bench_$tag.json 2> $OUT/bench_$tag.err
    timeout 600 ncu --metrics $M --clock-control none -k regex:k_scan_records -s 4 -c 1 --csv --log-file $OUT/ncu_$tag.csv \
      python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline $agg > $OUT/ncu_$tag.log 2>&1
    echo "$tag rc=$?"
  done
done
