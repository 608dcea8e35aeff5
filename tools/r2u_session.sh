#!/bin/bash
set -u
OUT=gpurun_out/r2u; mkdir -p $OUT
for lib in w1 stash; do
  FPX_LIB=$PWD/build/libfpx_$lib.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $OUT/s2_$lib python bench.py --config s2 --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo $lib rc=$?
done
