#!/bin/bash
# Drain warp with 19 x 42-plane rings (Ring1E): analyzer parity, A/B on C3;
# C2 ncu --set full with source + per-line instruction profile (producer).
set -u
O=gpurun_out/r2v7; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py tests/test_gpu_fullsize_configs.py -m gpu -q --timeout 300 -x -k "flow or FLOW or c3" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
TAG=r2v7/ab LIBS="build/libfpx_noeq.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c3" ROUNDS=4 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 3 -c 1 -o $O/full_c2 \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > $O/full_c2.log 2>&1; echo "full c2 rc=$?"
python tools/line_profile.py $O/full_c2.ncu-rep paper_conf_hpdc_lilfslg23_b200/libfpx.so k_scan_records --top 80 > $O/lines_c2.txt 2>&1
python tools/line_profile.py $O/full_c2.ncu-rep paper_conf_hpdc_lilfslg23_b200/libfpx.so k_scan_records --top 40 --outer > $O/lines_outer_c2.txt 2>&1
head -20 $O/lines_outer_c2.txt
