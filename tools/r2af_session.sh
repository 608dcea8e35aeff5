#!/bin/bash
# table_add: CAS on the home slot first (cas1) vs load-then-CAS (cas0)
set -u
TAG=r2af LIBS="build/libfpx_cas0.so;build/libfpx_cas1.so" CONFIGS="c1;c3;s1;s2;c2" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
