#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for t in 0 1 2 4; do
  timeout 600 python bench.py --steps 300 --warmup 10 --workload powerlaw1m --hybrid $t --no-cpu-baseline --no-variants > gpurun_out/hy_pl_$t.json 2> gpurun_out/hy_pl_$t.err
  timeout 900 python bench.py --steps 100 --warmup 5 --workload rmat22 --hybrid $t --no-cpu-baseline --no-variants > gpurun_out/hy_r22_$t.json 2> gpurun_out/hy_r22_$t.err
done
timeout 1200 python bench.py --steps 30 --warmup 3 --workload rmat25 --hybrid 2 --no-cpu-baseline --no-variants > gpurun_out/hy_r25_2.json 2> gpurun_out/hy_r25_2.err
echo done
