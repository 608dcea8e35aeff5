#!/bin/bash
# Per-library, per-config: warp instructions, duration and issue activity of
# one record-scan launch (ncu), plus an interleaved bench A/B.
#   TAG=x LIBS="a.so;b.so" CONFIGS="c2;c3" bash tools/ab_ncu_inst.sh
set -u
O=gpurun_out/${TAG:-abinst}; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
IFS=';' read -ra L <<< "$LIBS"
IFS=';' read -ra C <<< "$CONFIGS"
M=gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_elapsed
for cfg in "${C[@]}"; do for lib in "${L[@]}"; do
  n=$(basename $lib .so)
  FPX_LIB=$PWD/$lib timeout 600 ncu --metrics $M --clock-control none -k regex:k_scan_ -s 4 -c 1 --csv --log-file $O/ncu_${cfg}_$n.csv python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  python - $O/ncu_${cfg}_$n.csv $cfg $n <<'PY'
import csv,sys
rows=[r for r in csv.reader(open(sys.argv[1])) if len(r)>5]
h=rows[0]; v={r[h.index('Metric Name')]:r[h.index('Metric Value')] for r in rows[1:]}
print(f"ncu {sys.argv[2]:5s} {sys.argv[3]:14s} inst {int(v.get('smsp__inst_executed.sum','0').replace(',',''))/1e6:9.1f} M  time {v.get('gpu__time_duration.sum')} ns  issue {v.get('smsp__issue_active.avg.pct_of_peak_sustained_elapsed')} %")
PY
done; done
TAG=${TAG:-abinst} bash tools/ab_lib.sh 2>&1 | grep -v Traceback
