#!/bin/bash
# Sparse DEST kernel on the 24-warp x 32-plane ring for large traces
# (FPX_DEST_RING=3): A/B on C5 / C2 / C4a.
set -u
O=gpurun_out/r2v23; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
TAG=r2v23/ab LIBS="paper_conf_hpdc_lilfslg23_b200/libfpx.so;build/libfpx_dring3.so" CONFIGS="c5;c2;c4a" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
