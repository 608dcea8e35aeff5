#!/bin/bash
# Storm counting (count4_fp32): DEST parity suites, A/B against the previous
# counting (build/libfpx_cnt0.so), S1 / S2 ncu --set full with source and the
# per-line instruction profile of the storm kernel.
set -u
O=gpurun_out/r2v5; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py -m gpu -q --timeout 600 > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
TAG=r2v5/ab LIBS="build/libfpx_cnt0.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="s1;s2;c1" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
for cfg in s1 s2; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $O/full_$cfg \
    python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > $O/full_$cfg.log 2>&1; echo "full $cfg rc=$?"
  python tools/line_profile.py $O/full_$cfg.ncu-rep paper_conf_hpdc_lilfslg23_b200/libfpx.so k_scan_records --top 60 > $O/lines_$cfg.txt 2>&1
  python tools/line_profile.py $O/full_$cfg.ncu-rep paper_conf_hpdc_lilfslg23_b200/libfpx.so k_scan_records --top 40 --outer > $O/lines_outer_$cfg.txt 2>&1
  head -30 $O/lines_outer_$cfg.txt
done
