#!/bin/bash
# Sparse DEST kernel on 18 warps x 46-plane stages (Ring4, FPX_DEST_RING=4):
# DEST parity through that library, A/B on C2 / C5 / C4a against Ring1.
set -u
O=gpurun_out/r2v13; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
FPX_LIB=$PWD/build/libfpx_ring4.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_mixed.py tests/test_gpu_fullsize_configs.py -m gpu -q --timeout 300 -x -k "not flow and not FLOW and not c3" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
TAG=r2v13/ab LIBS="paper_conf_hpdc_lilfslg23_b200/libfpx.so;build/libfpx_ring4.so" CONFIGS="c2;c5;c4a" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
