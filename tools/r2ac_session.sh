#!/bin/bash
# C3 bisection over the round's commits at one fixed work split (75 % static, 256-record chunks)
set -u
export FPX_STATIC_PCT=75 FPX_DYN_CHUNK=256 FPX_TAIL_TILES=8
TAG=r2acb LIBS="build/libfpx_r1.so;build/libfpx_bis_1059e99.so;build/libfpx_bis_897e516.so;build/libfpx_bis_bc65ce0.so;build/libfpx_bis_8f54c98.so;build/libfpx_bis_99fc4ab.so;build/libfpx_bis_1c86888.so;build/libfpx_bis_5d55cf2.so;build/libfpx_bis_f62e8bc.so;build/libfpx_bis_8fe657a.so;build/libfpx_bis_8442200.so" CONFIGS="c3" ROUNDS=2 BENCH_ARGS="--steps 100" bash tools/ab_lib.sh
