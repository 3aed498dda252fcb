#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x --timeout 900 -k "ablations" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for dec in slots mma; do
  SPADEN_DECODE=$dec timeout 600 python bench.py --steps 500 --warmup 10 --dtype fp16 --no-cpu-baseline --no-cusparse --no-variants > gpurun_out/tc_$dec.json 2> gpurun_out/tc_$dec.err
done
SPADEN_DECODE=mma timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o gpurun_out/prof_mma python bench.py --steps 10 --warmup 3 --dtype fp16 --no-cpu-baseline --no-cusparse --no-variants > gpurun_out/ncu_mma.log 2>&1
echo done
