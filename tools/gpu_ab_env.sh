#!/bin/bash
# A/B of environment settings: ENVS="A=1 B=2;A=0" (';'-separated sets), fem1p5m kernel ms fp32/fp16
mkdir -p gpurun_out/ab; rm -f gpurun_out/ab/summary.txt
IFS=';' read -ra SETS <<< "${ENVS}"
for rep in 1 2; do
for dt in fp32 fp16; do
for e in "${SETS[@]}"; do
  env $e timeout 300 python bench.py --steps 1000 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" ${ARGS} > gpurun_out/ab/b.json 2> gpurun_out/ab/b.err
  python -c "import json; d=json.load(open('gpurun_out/ab/b.json')); print('$dt', '[$e]', round(d['roofline']['kernel_ms'],4), round(d['roofline']['frac'],3))" >> gpurun_out/ab/summary.txt 2>&1
done; done; done
cat gpurun_out/ab/summary.txt
