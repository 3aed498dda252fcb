#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x --timeout 900 -k "hybrid or pagerank or long" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for t in 1 2; do
  timeout 600 python bench.py --steps 300 --warmup 10 --workload powerlaw1m --hybrid $t --no-cpu-baseline --no-variants > gpurun_out/hy_pl_$t.json 2> gpurun_out/hy_pl_$t.err
  timeout 900 python bench.py --steps 100 --warmup 5 --workload rmat22 --hybrid $t --no-cpu-baseline --no-variants > gpurun_out/hy_r22_$t.json 2> gpurun_out/hy_r22_$t.err
done
timeout 1200 python bench.py --steps 30 --warmup 3 --workload rmat25 --hybrid 1 --no-cpu-baseline --no-variants > gpurun_out/hy_r25_1.json 2> gpurun_out/hy_r25_1.err
timeout 900 ncu --set full --clock-control none -k regex:k_residual -s 3 -c 1 -o gpurun_out/prof_res python bench.py --steps 5 --warmup 3 --workload rmat22 --hybrid 1 --no-cpu-baseline --no-variants --no-cusparse > gpurun_out/ncu_res.log 2>&1
echo done
