#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for dt in fp32 fp16; do
  SPADEN_KERNEL=v1 timeout 600 python bench.py --steps 1000 --warmup 10 --dtype $dt --no-cpu-baseline > gpurun_out/bench_v1_$dt.json 2> gpurun_out/bench_v1_$dt.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_v1 -s 5 -c 1 -o gpurun_out/prof_v1_fp32 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-cusparse > gpurun_out/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_v1 -s 5 -c 1 -o gpurun_out/prof_v1_fp16 python bench.py --steps 10 --warmup 3 --dtype fp16 --no-cpu-baseline --no-cusparse >> gpurun_out/ncu_full.log 2>&1
echo done
