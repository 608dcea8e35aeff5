#!/bin/bash
set -u
TAG=r2z LIBS="build/libfpx_w0f.so;build/libfpx_ss1.so" CONFIGS="s1;s2" ROUNDS=2 bash tools/ab_lib.sh
TAG=r2z ENVS="FPX_SCHED=1;FPX_DYN_CHUNK=128;FPX_DYN_CHUNK=64;FPX_TAIL_TILES=24;FPX_DYN_CHUNK=64 FPX_TAIL_TILES=24;FPX_STATIC_PCT=30 FPX_DYN_CHUNK=64 FPX_TAIL_TILES=24" ROUNDS=3 BENCH_ARGS="--config c3 --steps 100" bash tools/ab_env.sh
