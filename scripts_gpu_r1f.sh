#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 500 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 900 python bench.py --steps 200 --warmup 5 --workload rmat22 --no-cpu-baseline > gpurun_out/bench_rmat22.json 2> gpurun_out/bench_rmat22.err
timeout 1200 python bench.py --steps 50 --warmup 3 --workload rmat25 --cpu-seconds 5 > gpurun_out/bench_rmat25.json 2> gpurun_out/bench_rmat25.err
timeout 600 python bench.py --impl reference --steps 50 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
echo done
