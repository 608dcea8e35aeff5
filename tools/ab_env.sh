#!/bin/bash
# A/B of environment settings (e.g. FPX_RING) on one build, interleaved.
#   ENVS="FPX_RING=0;FPX_RING=1" ROUNDS=3 BENCH_ARGS="--steps 200" bash tools/ab_env.sh
set -u
OUT=gpurun_out/${TAG:-abenv}; mkdir -p $OUT
python __graft_entry__.py build > /dev/null 2>&1
bash tools/build_tuning.sh && export FPX_LIB=$PWD/build/libfpx_tuning.so
IFS=';' read -ra V <<< "$ENVS"
for r in $(seq 1 ${ROUNDS:-3}); do
  for i in "${!V[@]}"; do
    env ${V[$i]} timeout 300 python bench.py --no-e2e --no-cpu-baseline ${BENCH_ARGS:-} > $OUT/ab_${i}_$r.json 2>> $OUT/ab.err
    python -c "import json; d=json.loads(open('$OUT/ab_${i}_$r.json').read()); print('env ${V[$i]} round $r', round(d['roofline']['achieved']), 'GB/s', d['clocks']['sm_mhz'])"
  done
done
