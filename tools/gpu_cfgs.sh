#!/bin/bash
# fem1p5m kernel ms per tile config (fp32 + fp16), plus a parity check of the configs
mkdir -p gpurun_out/cfgs; rm -f gpurun_out/cfgs/summary.txt
timeout 600 python tools/cfg_check.py ${CHECK:-2,15} > gpurun_out/cfgs/check.log 2>&1; echo "check rc=$?" >> gpurun_out/cfgs/check.log
for dt in fp32 fp16; do
for cfg in ${CFGS:-2 15 5 7 3 1 14}; do
  SPADEN_TILE_CFG=$cfg timeout 300 python bench.py --steps 1000 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/cfgs/b_${cfg}_$dt.json 2> gpurun_out/cfgs/b_${cfg}_$dt.err
  python -c "import json; d=json.load(open('gpurun_out/cfgs/b_${cfg}_$dt.json')); print('$dt', $cfg, round(d['roofline']['kernel_ms'],4), round(d['roofline']['frac'],3))" >> gpurun_out/cfgs/summary.txt 2>&1
done; done
cat gpurun_out/cfgs/summary.txt
