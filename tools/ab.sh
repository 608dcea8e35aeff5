#!/bin/bash
# A/B kernel variants on one box: build libfpx.so with extra -D flags per
# variant into build/ab_<i>.so, then run the bench interleaved (A B A B ...)
# so that power-cap drift hits every variant alike.
#   VARIANTS="-DX=1;-DX=2" ROUNDS=3 BENCH_ARGS="--steps 200" bash tools/ab.sh
set -u
OUT=gpurun_out/${TAG:-ab}; mkdir -p $OUT build
python __graft_entry__.py build > /dev/null 2>&1
IFS=';' read -ra V <<< "$VARIANTS"
SRC="paper_conf_hpdc_lilfslg23_b200/csrc/fpx_api.cu paper_conf_hpdc_lilfslg23_b200/csrc/fpx_scan_records.cu paper_conf_hpdc_lilfslg23_b200/csrc/fpx_scan_tensor.cu paper_conf_hpdc_lilfslg23_b200/csrc/fpx_table.cu"
for i in "${!V[@]}"; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O3 -shared -Iinclude ${V[$i]} $SRC -o build/ab_$i.so &
done
wait
for r in $(seq 1 ${ROUNDS:-3}); do
  for i in "${!V[@]}"; do
    FPX_LIB=$PWD/build/ab_$i.so timeout 300 python bench.py --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} > $OUT/ab_${i}_$r.json 2>> $OUT/ab.err
    python -c "import json,sys; d=json.loads(open('$OUT/ab_${i}_$r.json').read()); print('variant $i (${V[$i]}) round $r', round(d['roofline']['achieved']), 'GB/s', d['clocks']['sm_mhz'])"
  done
done
