#!/bin/bash
set -u
python __graft_entry__.py build > /dev/null 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_mixed.py tests/test_gpu_live.py -m gpu -x -q > gpurun_out/r2ag_pytest.log 2>&1; echo pytest rc=$?; tail -2 gpurun_out/r2ag_pytest.log
TAG=r2ag LIBS="build/libfpx_cas0.so;build/libfpx_cas2.so" CONFIGS="c1;c3;s2;c2" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
