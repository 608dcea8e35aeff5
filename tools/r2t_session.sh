#!/bin/bash
# storm kernel with the header stash: parity, then A/B against the previous storm kernel (warm 8 / warm 1)
set -u
OUT=gpurun_out/${TAG:-r2t}; mkdir -p $OUT
python __graft_entry__.py build > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py -m gpu -x -q -k "storm or dense or zoo or noagg" > $OUT/pytest.log 2>&1; echo pytest rc=$? ; tail -3 $OUT/pytest.log
TAG=${TAG:-r2t} LIBS="build/libfpx_w8.so;build/libfpx_w1.so;build/libfpx_stash.so" CONFIGS="s1;s2;c1" ROUNDS=2 bash tools/ab_lib.sh
