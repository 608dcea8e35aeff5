#!/bin/bash
set -u
OUT=gpurun_out/r2y; mkdir -p $OUT
python __graft_entry__.py build > $OUT/build.log 2>&1
cp paper_conf_hpdc_lilfslg23_b200/libfpx.so $OUT/
for cfg in s2 s1 c2; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $OUT/full_$cfg python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo $cfg rc=$?
done
