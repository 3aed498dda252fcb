#!/bin/bash
# gpu_cfg_sweep.sh "cfgs": fem1p5m kernel ms per SPADEN_TILE_CFG, fp32 and fp16, twice
mkdir -p gpurun_out
: > gpurun_out/cfg.txt
for rep in 1 2; do for cfg in $1; do for dt in fp32 fp16; do
  SPADEN_TILE_CFG=$cfg timeout 600 python bench.py --steps 1000 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/cfg_${cfg}_$dt.json 2> gpurun_out/cfg_${cfg}_$dt.err
  python -c "import json; d=json.load(open('gpurun_out/cfg_${cfg}_$dt.json')); print('cfg $cfg $dt', round(d['roofline']['kernel_ms'],4))" >> gpurun_out/cfg.txt 2>&1
done; done; done
cat gpurun_out/cfg.txt
