#!/bin/bash
# Storm kernel with emit_kinds_cta inlined (FPX_EMIT_INLINE): storm parity
# through that library, A/B on S1 / S2.
set -u
O=gpurun_out/r2v17; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
FPX_LIB=$PWD/build/libfpx_emitinl.so timeout 900 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py -m gpu -q --timeout 300 -x -k "storm or dense or cta" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
TAG=r2v17/ab LIBS="paper_conf_hpdc_lilfslg23_b200/libfpx.so;build/libfpx_emitinl.so" CONFIGS="s1;s2" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
