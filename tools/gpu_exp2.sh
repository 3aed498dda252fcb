#!/bin/bash
# gpu_exp2.sh "libs" "cfgs" [dtype]: kernel_ms per (lib variant, SPADEN_TILE_CFG)
mkdir -p gpurun_out
: > gpurun_out/exp2.txt
dt=${3:-fp32}
for v in $1; do for c in $2; do
  SPADEN_TILE_CFG=$c SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 300 python bench.py --steps 500 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/e2.json 2> gpurun_out/e2_${v}_$c.err
  python -c "import json; d=json.load(open('gpurun_out/e2.json')); print('$v cfg$c $dt', round(d['roofline']['kernel_ms'],5))" >> gpurun_out/exp2.txt 2>&1
done; done
cat gpurun_out/exp2.txt
