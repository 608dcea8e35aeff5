set -u
mkdir -p gpurun_out/r2e
python __graft_entry__.py build > gpurun_out/r2e/build.log 2>&1 || { tail -30 gpurun_out/r2e/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py -m gpu -x -q --timeout 600 -k "zoo or storm or worked or brute or synthetic" > gpurun_out/r2e/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r2e/pytest.log
TAG=r2e LIBS="build/libfpx_r1.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so;build/libfpx_ind.so;build/libfpx_noct.so;build/libfpx_allct.so" CONFIGS="c1;s1;s2;c3;c2" ROUNDS=2 BENCH_ARGS="--steps 60" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
