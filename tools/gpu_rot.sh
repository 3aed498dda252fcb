#!/bin/bash
# row-rotation experiment: parity (bitwise vs SPADEN_ROT=0 config), fem1p5m times with/without, ncu wavefronts
mkdir -p gpurun_out/rot
timeout 600 python tools/cfg_check.py ${CHECK:-2,15,5,3} > gpurun_out/rot/check.log 2>&1; echo "check rc=$?" >> gpurun_out/rot/check.log
SPADEN_ROT=0 timeout 600 python tools/cfg_check.py ${CHECK:-2,15} > gpurun_out/rot/check_norot.log 2>&1; echo "check rc=$?" >> gpurun_out/rot/check_norot.log
for dt in fp32 fp16; do
for rot in 1 0; do
  SPADEN_ROT=$rot timeout 300 python bench.py --steps 1000 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/rot/b_${rot}_$dt.json 2> gpurun_out/rot/b_${rot}_$dt.err
  python -c "import json; d=json.load(open('gpurun_out/rot/b_${rot}_$dt.json')); print('$dt rot=$rot', round(d['roofline']['kernel_ms'],4), round(d['roofline']['frac'],3), 'conv', round(d['convert']['ns_per_nnz'],3))" >> gpurun_out/rot/summary.txt 2>&1
done; done
for dt in fp32 fp16; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o gpurun_out/rot/rot_$dt python bench.py --steps 10 --warmup 3 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/rot/ncu_$dt.log 2>&1
done
cat gpurun_out/rot/summary.txt
