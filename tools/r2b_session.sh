set -u
mkdir -p gpurun_out/r2b
python __graft_entry__.py build > gpurun_out/r2b/build.log 2>&1 || { tail -30 gpurun_out/r2b/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_live.py tests/test_gpu_hooks.py tests/test_gpu_parity.py tests/test_bench.py -m gpu -x -q --timeout 600 > gpurun_out/r2b/pytest.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/r2b/pytest.log
TAG=r2b LIBS="build/libfpx_r1.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="s1;s2;c2;c3;c1" ROUNDS=2 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
