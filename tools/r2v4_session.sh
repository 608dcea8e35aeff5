#!/bin/bash
# FLOW candidate filter: parity (analyzer suites), A/B on C3 against the
# unfiltered build, warp spread on C3.
set -u
O=gpurun_out/r2v4; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py tests/test_gpu_fullsize_configs.py -m gpu -q --timeout 600 -k "flow or FLOW or c3 or zoo" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
TAG=r2v4/ab LIBS="build/libfpx_nocand.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c3;c2" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
timeout 600 python tools/warp_times.py c3 > $O/warp_times.txt 2>&1; grep -E "^c[0-9]|exact path" $O/warp_times.txt
