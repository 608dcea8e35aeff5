#!/bin/bash
# Static share of the DEST work split (75 / 60 / 50 %) on this box, its slow-SM
# profile (warp spread), and the analyzer live / FETCH_NEW test.
set -u
O=gpurun_out/r2v12; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_live.py -m gpu -q --timeout 300 > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 900 python tools/warp_times.py c2 c3 c5 > $O/warp_times.txt 2>&1; grep -E "^c[0-9]|exact path" $O/warp_times.txt
TAG=r2v12/ab LIBS="paper_conf_hpdc_lilfslg23_b200/libfpx.so;build/libfpx_st60.so;build/libfpx_st50.so" CONFIGS="c2;c5" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
