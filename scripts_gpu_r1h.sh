#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for cfg in 2 3 7 8 9; do
  SPADEN_TILE_CFG=$cfg timeout 600 python bench.py --steps 500 --warmup 10 --workload fem62k --no-cpu-baseline --no-cusparse > gpurun_out/sw62_${cfg}.json 2> gpurun_out/sw62_${cfg}.err
done
timeout 600 python bench.py --steps 500 --warmup 10 --workload fem62k --no-cpu-baseline > gpurun_out/bench_fem62k.json 2> gpurun_out/bench_fem62k.err
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
echo done
