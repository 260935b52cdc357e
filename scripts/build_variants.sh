#!/bin/bash
# experiment builds of the library (compile-time switches), loaded via SZX_LIB
cd "$(dirname "$0")/.."
mkdir -p build_exp
for v in "$@"; do
  name=$(echo "$v" | tr ' =-' '___')
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -fmad=false --ftz=false \
    -shared -Xcompiler -fPIC -cudart static $v -o build_exp/lib_$name.so paper_conf_hpdc_yudztt0c22_b200/csrc/szx_api.cu &
done
wait
ls build_exp
