#!/bin/bash
set -u
TAG=r2ai LIBS="build/libfpx_pol0.so;build/libfpx_pol1.so" CONFIGS="c2;c5;c3" bash tools/ab_ncu_inst.sh
TAG=r2ai LIBS="build/libfpx_pol0.so;build/libfpx_pol1.so;build/libfpx_r1.so" CONFIGS="c2;c5;c4a;c3;c1" ROUNDS=3 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
