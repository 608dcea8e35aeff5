#!/bin/bash
# Tuning build of libfpx (-DFPX_TUNING: launch-shape knobs read from the
# environment, see fpx_scan_records.cu Tuning) at build/libfpx_tuning.so; the
# A/B scripts point the binding at it with FPX_LIB.  Never the product library.
set -eu
mkdir -p build
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O3 -shared \
  -DFPX_TUNING -I include paper_conf_hpdc_lilfslg23_b200/csrc/*.cu -o build/libfpx_tuning.so
