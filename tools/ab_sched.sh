#!/bin/bash
# Record-scan load balance: parity tests, per-warp end-time spread
# (tools/warp_times.py) and an interleaved A/B of scheduler settings given as
# environment assignments (FPX_SCHED, FPX_STATIC_PCT; fpx_scan_records.cu).
#   TAG=dyn3 ENVS="FPX_STATIC_PCT=75;FPX_STATIC_PCT=50" CFGS="c2 c3" ROUNDS=2 TESTS=0 bash tools/ab_sched.sh
set -u
O=gpurun_out/${TAG:-dyn}; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -20 $O/build.log; exit 1; }
bash tools/build_tuning.sh && export FPX_LIB=$PWD/build/libfpx_tuning.so
if [ "${TESTS:-1}" = 1 ]; then
  timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_fullsize_configs.py -x -q --timeout 600 > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -5 $O/pytest.log
fi
if [ "${WT:-1}" = 1 ]; then
  timeout 300 python tools/warp_times.py ${CFGS:-c2 c4a c5 c3} > $O/warp_times.txt 2>&1; grep -v "^ \|Remark\|warning" $O/warp_times.txt
fi
IFS=';' read -ra V <<< "${ENVS:-FPX_SCHED=0;FPX_SCHED=1}"
for r in $(seq 1 ${ROUNDS:-2}); do for cfg in ${CFGS:-c2 c4a c5 c3}; do for i in "${!V[@]}"; do
  env ${V[$i]} timeout 300 python bench.py --config $cfg --steps ${STEPS:-100} --no-e2e --no-cpu-baseline > $O/ab_${cfg}_${i}_$r.json 2>>$O/ab.err
  python -c "import json; d=json.loads(open('$O/ab_${cfg}_${i}_$r.json').read()); print('$cfg ${V[$i]} r$r', round(d['roofline']['achieved']), 'GB/s', round(d['roofline']['kernel_ms'],4),'ms', d['clocks']['sm_mhz'], d['clocks']['reasons'])"
done; done; done
