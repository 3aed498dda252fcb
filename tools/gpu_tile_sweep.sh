#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for cfg in 1 2 3 5 6 7; do for dt in fp32 fp16; do
  SPADEN_TILE_CFG=$cfg timeout 600 python bench.py --steps 500 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse > gpurun_out/sw_${cfg}_$dt.json 2> gpurun_out/sw_${cfg}_$dt.err
done; done
SPADEN_TILE_CFG=3 timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o gpurun_out/prof_h3_fp32 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-cusparse > gpurun_out/ncu_full.log 2>&1
echo done
