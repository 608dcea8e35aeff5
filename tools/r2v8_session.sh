#!/bin/bash
# Full GPU suite + smoke + compute-sanitizer (memcheck / racecheck / synccheck /
# initcheck) over tools/sanitize.py on the current build.
set -u
O=gpurun_out/r2v8; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
timeout 600 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
bash tools/sanitize_all.sh $O/sanitizer
