#!/bin/bash
# A/B variant build of libfpx: build/libfpx_<name>.so with extra nvcc flags
# (compile-time switches of the kernels), for tools/ab_lib.sh.
#   bash tools/build_variant.sh name -DFPX_DENSE_EVENTS=33 ...
set -eu
name=$1; shift
mkdir -p build
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O3 -shared \
  -I include "$@" paper_conf_hpdc_lilfslg23_b200/csrc/*.cu -o build/libfpx_$name.so
