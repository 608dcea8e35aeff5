#!/bin/bash
set -u
OUT=gpurun_out/r2v; mkdir -p $OUT
TAG=r2v LIBS="build/libfpx_w1.so;build/libfpx_stash2.so" CONFIGS="s1;s2;c2;c1" ROUNDS=2 bash tools/ab_lib.sh
FPX_LIB=$PWD/build/libfpx_stash2.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $OUT/s2_stash2 python bench.py --config s2 --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo rc=$?
