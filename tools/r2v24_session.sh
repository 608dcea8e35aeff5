#!/bin/bash
# One-plane DEST traces on the 24-warp ring (FPX_ONE_PLANE_RING): parity
# (DEST suites, full-size C5 / C4a / C2), A/B C5 / C2 / C4a / S1 against
# build/libfpx_op0.so.
set -u
O=gpurun_out/r2v24; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_mixed.py tests/test_gpu_fullsize_configs.py tests/test_gpu_fullsize.py -m gpu -q --timeout 900 -x -k "not flow and not FLOW and not c3" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
TAG=r2v24/ab LIBS="build/libfpx_op0.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c5;c2;c4a;s1" ROUNDS=2 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
