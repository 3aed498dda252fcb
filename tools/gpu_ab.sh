#!/bin/bash
mkdir -p gpurun_out
for v in base el na base el na; do for dt in fp32 fp16; do
  SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 600 python bench.py --steps 1000 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants > gpurun_out/ab_${v}_$dt.json 2> gpurun_out/ab_${v}_$dt.err
  python -c "import json; d=json.load(open('gpurun_out/ab_${v}_$dt.json')); print('$v $dt', d['roofline']['kernel_ms'])" >> gpurun_out/ab.txt
done; done
echo done
