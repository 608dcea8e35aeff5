#!/bin/bash
# FLOW exact path: pointer call (fi0) vs inlined lean path (fi1) vs inlined record path (fi2), C3
set -u
TAG=r2ad LIBS="build/libfpx_r1.so;build/libfpx_fi0.so;build/libfpx_fi1.so;build/libfpx_fi2.so" CONFIGS="c3" ROUNDS=2 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
export FPX_STATIC_PCT=75 FPX_DYN_CHUNK=256 FPX_TAIL_TILES=8
echo "fixed split 75/256"
TAG=r2ad2 LIBS="build/libfpx_r1.so;build/libfpx_fi0.so;build/libfpx_fi1.so;build/libfpx_fi2.so" CONFIGS="c3" ROUNDS=2 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
