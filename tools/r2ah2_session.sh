#!/bin/bash
set -u
python __graft_entry__.py build > /dev/null 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_mixed.py -m gpu -x -q -k "storm or dense" > gpurun_out/r2ah2_pytest.log 2>&1; echo pytest rc=$?; tail -2 gpurun_out/r2ah2_pytest.log
TAG=r2ah2 LIBS="build/libfpx_nl0.so;build/libfpx_nl1.so" CONFIGS="s1;s2;c1" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
