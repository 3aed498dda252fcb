#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x --timeout 900 -k "ablations or bitwise_equal" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for dec in slots quad pair; do for dt in fp32 fp16; do
  SPADEN_DECODE=$dec timeout 600 python bench.py --steps 500 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants > gpurun_out/lpb_${dec}_$dt.json 2> gpurun_out/lpb_${dec}_$dt.err
done; done
SPADEN_DECODE=quad timeout 900 ncu --set full --clock-control none -k regex:spmv_tiled -s 5 -c 1 -o gpurun_out/prof_quad16 python bench.py --steps 10 --warmup 3 --dtype fp16 --no-cpu-baseline --no-cusparse --no-variants > gpurun_out/ncu_q.log 2>&1
echo done
