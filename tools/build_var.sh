#!/bin/bash
# Build a variant of libdts.so with extra nvcc flags: tools/build_var.sh NAME [-DFOO ...]
cd "$(dirname "$0")/.."
NAME=$1; shift
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared -Xptxas -O3 "$@" \
  -I include -o paper_conf_ipps_gonthiermt22_b200/lib/var_$NAME.so paper_conf_ipps_gonthiermt22_b200/csrc/*.cu
