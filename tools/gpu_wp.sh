#!/bin/bash
# warp-private kernel experiment: parity across configs, then fem1p5m kernel ms per config
mkdir -p gpurun_out/wp
timeout 600 python tools/cfg_check.py ${CHECK:-2,15,20,21,22,23,24,25,26,27} > gpurun_out/wp/check.log 2>&1; echo "check rc=$?" >> gpurun_out/wp/check.log
for dt in fp32 fp16; do
for cfg in ${CFGS:-2 15 20 21 22 23 24 25 26 27}; do
  SPADEN_TILE_CFG=$cfg timeout 300 python bench.py --steps 500 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/wp/b_${cfg}_$dt.json 2> gpurun_out/wp/b_${cfg}_$dt.err
  python -c "import json; d=json.load(open('gpurun_out/wp/b_${cfg}_$dt.json')); print('$dt', $cfg, round(d['roofline']['kernel_ms'],4), round(d['roofline']['frac'],3))" >> gpurun_out/wp/summary.txt 2>&1
done; done
cat gpurun_out/wp/summary.txt
