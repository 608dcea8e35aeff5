#!/bin/bash
# storm kernel knobs: warm threshold (w8 / w1 / w0) and ring geometry (tuning build)
set -u
OUT=gpurun_out/${TAG:-r2s}; mkdir -p $OUT
TAG=${TAG:-r2s} LIBS="build/libfpx_w8.so;build/libfpx_w1.so;build/libfpx_w0.so" CONFIGS="s1;s2" ROUNDS=2 bash tools/ab_lib.sh
for cfg in s1 s2; do for r in 1 2; do for ring in 1 0 2; do
  FPX_RING=$ring FPX_LIB=$PWD/build/libfpx_tuning.so timeout 300 python bench.py --no-e2e --no-cpu-baseline --config $cfg > $OUT/ring_${cfg}_${ring}_$r.json 2>> $OUT/ab.err
  python -c "import json; d=json.loads(open('$OUT/ring_${cfg}_${ring}_$r.json').read()); print('$cfg ring $ring round $r', round(d['roofline']['achieved']), 'GB/s kernel_ms', round(d['roofline']['kernel_ms'],4), d['clocks']['sm_mhz'])"
done; done; done
