#!/bin/bash
# CTA table: first sightings counted in shared memory and inserted by the
# CTA's last warp (FPX_CT_DEFER_FIRST=1): storm parity through that library,
# A/B on S1 / S2.
set -u
O=gpurun_out/r2v21; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
FPX_LIB=$PWD/build/libfpx_defer.so timeout 1200 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py -m gpu -q --timeout 600 -x -k "storm or dense or cta or zoo" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
TAG=r2v21/ab LIBS="paper_conf_hpdc_lilfslg23_b200/libfpx.so;build/libfpx_defer.so" CONFIGS="s1;s2" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
