#!/bin/bash
# gpu_ncu_exp.sh "variants" [dtype]: one ncu --set full capture of k_spmv_tiled per exp/libspaden_<v>.so
mkdir -p gpurun_out
dt=${2:-fp32}
for v in $1; do
  SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o gpurun_out/px_${v}_$dt -f python bench.py --steps 10 --warmup 3 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/px_${v}.log 2>&1
done
ls -la gpurun_out/px_*
