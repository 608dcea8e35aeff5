#!/bin/bash
# Last check of round 2 (after the deferred first sightings): GPU suite, smoke,
# headline bench, storm bench lines + atomics.
set -u
T=r2fin4; O=gpurun_out/$T; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { echo BUILD FAILED; tail -30 $O/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
timeout 600 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; echo "bench c2 rc=$?"; cut -c1-200 $O/bench_c2.json
TAG=$T/storm CFGS="s1 s2 c2" bash tools/storm_ncu.sh
