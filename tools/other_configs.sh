#!/bin/bash
# Bench line of every non-headline config (JSON lines to stdout).
for c in ${CONFIGS:-c1 c3 c4a c4b c4b16 s1 s2 c5}; do
  timeout 600 python bench.py --config $c --steps ${STEPS:-50} --warmup 3 --no-e2e
done
