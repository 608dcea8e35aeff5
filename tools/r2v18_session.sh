#!/bin/bash
# The CTA table's returning-add path (storm launches > 2^24 records) and the
# whole parity file.
set -u
O=gpurun_out/r2v18; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 900 > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
grep -E "large_launch|FAILED|Error" $O/pytest.log | head
