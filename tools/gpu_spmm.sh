#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x --timeout 900 -k "spmm" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 500 --spmm 2,4,8 --no-cpu-baseline > gpurun_out/bench_spmm.json 2> gpurun_out/bench_spmm.err
timeout 900 python bench.py --steps 500 --spmm 2,4,8 --dtype fp16 --no-cpu-baseline --no-variants > gpurun_out/bench_spmm16.json 2> gpurun_out/bench_spmm16.err
echo done
