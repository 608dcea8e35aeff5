#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck over tools/sanitize.py.
OUT=${1:-gpurun_out/sanitizer}
mkdir -p $OUT
for t in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $t --error-exitcode 9 python tools/sanitize.py > $OUT/$t.txt 2>&1
  echo "$t rc=$?"; tail -2 $OUT/$t.txt
done
