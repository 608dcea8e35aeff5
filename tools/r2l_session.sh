set -u
O=gpurun_out/r2l; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
cp paper_conf_hpdc_lilfslg23_b200/libfpx.so $O/libfpx_box.so
timeout 1500 python -m pytest tests -m gpu -x -q --timeout 600 > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for cfg in c2 c3 c5; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $O/full_$cfg python bench.py --config $cfg --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "full $cfg rc=$?"
done
