#!/bin/bash
# A/B of prebuilt libraries (e.g. the previous commit's build/libfpx_old.so
# against the current build), interleaved, over several bench configs.
#   LIBS="build/libfpx_old.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c2;c1" ROUNDS=2 bash tools/ab_lib.sh
set -u
OUT=gpurun_out/${TAG:-ablib}; mkdir -p $OUT
python __graft_entry__.py build > /dev/null 2>&1
IFS=';' read -ra L <<< "$LIBS"
IFS=';' read -ra C <<< "$CONFIGS"
for cfg in "${C[@]}"; do
  for r in $(seq 1 ${ROUNDS:-2}); do
    for i in "${!L[@]}"; do
      FPX_LIB=$PWD/${L[$i]} timeout 300 python bench.py --no-e2e --no-cpu-baseline --config $cfg ${BENCH_ARGS:-} > $OUT/ab_${cfg}_${i}_$r.json 2>> $OUT/ab.err
      python -c "import json; d=json.loads(open('$OUT/ab_${cfg}_${i}_$r.json').read()); print('$cfg lib ${L[$i]} round $r', round(d['roofline']['achieved']), 'GB/s kernel_ms', round(d['roofline']['kernel_ms'],4), 'step_ms', round(d['ms_per_step'],4), d['clocks']['sm_mhz'])"
    done
  done
done
