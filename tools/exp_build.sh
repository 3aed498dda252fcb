#!/bin/bash
# exp_build.sh NAME [nvcc -D flags...]: build an experiment variant exp/libspaden_NAME.so
set -e
name=$1; shift
mkdir -p exp
cd "$(dirname "$0")/.."
/usr/local/cuda/bin/nvcc -O3 -std=c++17 -lineinfo -gencode arch=compute_100a,code=sm_100a \
  -Xcompiler -fPIC,-O2,-fvisibility=hidden --expt-relaxed-constexpr -cudart static -Xlinker --no-undefined "$@" \
  -I include -I paper_conf_icpp_cheny24_b200/csrc -shared paper_conf_icpp_cheny24_b200/csrc/*.cu -o exp/libspaden_$name.so
echo exp/libspaden_$name.so
