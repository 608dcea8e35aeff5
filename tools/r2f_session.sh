set -u
O=gpurun_out/r2f; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_mixed.py tests/test_gpu_parity.py tests/test_gpu_live.py -m gpu -x -q --timeout 600 > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
TAG=r2f LIBS="build/libfpx_r1.so;paper_conf_hpdc_lilfslg23_b200/libfpx.so" CONFIGS="c1;s1;s2;c3;c2;c5" ROUNDS=2 BENCH_ARGS="--steps 60" bash tools/ab_lib.sh 2>&1 | grep -v Traceback
M=gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum
for cfg in c2 c3 c5; do for L in build/libfpx_r1.so paper_conf_hpdc_lilfslg23_b200/libfpx.so; do
  n=$(basename $L .so)
  FPX_LIB=$PWD/$L timeout 600 ncu --metrics $M --clock-control none -k regex:k_scan_records -s 4 -c 1 --csv --log-file $O/ncu_${cfg}_$n.csv python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  python - $O/ncu_${cfg}_$n.csv $cfg $n <<'PY'
import csv,sys
rows=[r for r in csv.reader(open(sys.argv[1])) if len(r)>5]
h=rows[0]; vals={r[h.index('Metric Name')]:r[h.index('Metric Value')] for r in rows[1:]}
print(sys.argv[2], sys.argv[3], vals)
PY
done; done
for L in build/libfpx_r1.so paper_conf_hpdc_lilfslg23_b200/libfpx.so; do n=$(basename $L .so)
  FPX_LIB=$PWD/$L timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $O/full_c3_$n python bench.py --config c3 --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "full c3 $n rc=$?"
done
