set -u
mkdir -p gpurun_out/r2c
python __graft_entry__.py build > gpurun_out/r2c/build.log 2>&1 || { tail -30 gpurun_out/r2c/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_hooks.py tests/test_bench.py -m gpu -x -q --timeout 600 > gpurun_out/r2c/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2c/pytest.log
TAG=r2c LIBS="build/libfpx_r1.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c3;s1;s2;c1" ROUNDS=1 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
TAG=r2c CFGS="s1 s2 c3" FULL="s1 c3" bash tools/storm_ncu.sh
