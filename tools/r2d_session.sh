set -u
mkdir -p gpurun_out/r2d
python __graft_entry__.py build > gpurun_out/r2d/build.log 2>&1 || { tail -30 gpurun_out/r2d/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q --timeout 600 > gpurun_out/r2d/pytest.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/r2d/pytest.log
TAG=r2d LIBS="build/libfpx_r1.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="s1;s2;c3;c1;c2;c4a" ROUNDS=1 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
TAG=r2d CFGS="s1 s2" FULL="s1" bash tools/storm_ncu.sh
