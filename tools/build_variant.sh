#!/bin/bash
# usage: tools/build_variant.sh NAME [-DFLAG ...]   -> variants/lib_NAME.so (tuning only)
n=$1; shift
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared -cudart static "$@" \
  -o variants/lib_$n.so paper_conf_middleware_tanaabcrtn24_b200/csrc/ckpt.cu 2>&1 | grep -v "spill\|^$" 
echo "built $n"
