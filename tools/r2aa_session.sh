#!/bin/bash
set -u
OUT=gpurun_out/r2aa; mkdir -p $OUT
python __graft_entry__.py build > /dev/null 2>&1
for lib in r1 cur; do
  FPX_LIB=$PWD/build/libfpx_$lib.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $OUT/c3_$lib python bench.py --config c3 --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo $lib rc=$?
done
TAG=r2aa LIBS="build/libfpx_r1.so;build/libfpx_cur.so" CONFIGS="c3" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
TAG=r2aa ENVS="FPX_STATIC_PCT=45;FPX_STATIC_PCT=75;FPX_STATIC_PCT=75 FPX_DYN_CHUNK=256;FPX_SCHED=0" ROUNDS=3 BENCH_ARGS="--config c3 --steps 100" bash tools/ab_env.sh
