#!/bin/bash
# Where the storm kernel waits now: ncu --set full of S1 / S2 with source,
# per-line instructions and stall samples.
set -u
O=gpurun_out/r2v15; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for cfg in s1 s2; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $O/full_$cfg \
    python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > $O/full_$cfg.log 2>&1; echo "full $cfg rc=$?"
  python tools/line_profile.py $O/full_$cfg.ncu-rep paper_conf_hpdc_lilfslg23_b200/libfpx.so k_scan_records --top 50 --col "Warp Stall Sampling (All Samples)" > $O/stall_lines_$cfg.txt 2>&1
  python tools/line_profile.py $O/full_$cfg.ncu-rep paper_conf_hpdc_lilfslg23_b200/libfpx.so k_scan_records --top 30 --outer --col "Warp Stall Sampling (All Samples)" > $O/stall_outer_$cfg.txt 2>&1
  head -25 $O/stall_lines_$cfg.txt
done
