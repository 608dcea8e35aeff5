#!/bin/bash
# BF16 items in the FP16 lists (FPX_MERGE_HALVES) and storm headers loaded one
# iteration ahead (FPX_STORM_HPRE 2): parity (witness isolation, zoo, storms,
# full-size C4a), A/B C4a / C2 against build/libfpx_mh0.so and S1 / S2
# against build/libfpx_hpre1.so.
set -u
O=gpurun_out/r2v16; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py tests/test_gpu_fullsize_configs.py -m gpu -q --timeout 300 -x -k "not flow and not FLOW and not c3" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
TAG=r2v16/ab_mh LIBS="build/libfpx_mh0.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c4a;c2" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
TAG=r2v16/ab_hpre LIBS="build/libfpx_hpre1.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="s1;s2" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
