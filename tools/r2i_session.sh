set -u
O=gpurun_out/r2i; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py -m gpu -x -q --timeout 600 > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 600 python tools/warp_times.py c3 > $O/wt_cur.txt 2>&1; grep -E "^c[0-9]" $O/wt_cur.txt
TAG=r2i LIBS="build/libfpx_r1.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c3;s1;c1" ROUNDS=2 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
