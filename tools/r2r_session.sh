set -u
O=gpurun_out/r2r; mkdir -p $O/sanitizer
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "storm_cta" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool python tools/sanitize.py > $O/sanitizer/$tool.txt 2>&1; echo "$tool rc=$?"; tail -2 $O/sanitizer/$tool.txt
done
