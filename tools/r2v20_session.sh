#!/bin/bash
# Unroll of the storm exact path's class count (FPX_COUNT_UNROLL 2 / 4 / 8):
# A/B on S1 / S2 (+ storm parity through the 8x build).
set -u
O=gpurun_out/r2v20; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
FPX_LIB=$PWD/build/libfpx_cu8.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 600 -x -k "storm or dense" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
TAG=r2v20/ab LIBS="paper_conf_hpdc_lilfslg23_b200/libfpx.so;build/libfpx_cu8.so;build/libfpx_cu2.so" CONFIGS="s1;s2" ROUNDS=2 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
