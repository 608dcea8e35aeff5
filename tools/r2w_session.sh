#!/bin/bash
set -u
TAG=r2w LIBS="build/libfpx_w1b.so;build/libfpx_w1s.so;build/libfpx_w0s.so;build/libfpx_w2.so" CONFIGS="s1;s2" ROUNDS=2 bash tools/ab_lib.sh
