#!/bin/bash
# first GPU session: tests, smoke, bench, ncu
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt 2>&1
nproc >> gpurun_out/gpu.txt; python -c "import torch;p=torch.cuda.get_device_properties(0);print(p.name,p.multi_processor_count,p.L2_cache_size if hasattr(p,'L2_cache_size') else '')" >> gpurun_out/gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 1000 --warmup 10 > gpurun_out/bench_fp32.json 2> gpurun_out/bench_fp32.err
timeout 600 python bench.py --steps 1000 --warmup 10 --dtype fp16 --no-cpu-baseline > gpurun_out/bench_fp16.json 2> gpurun_out/bench_fp16.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 30 -c 60 --csv --log-file gpurun_out/launches_fp32.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv -s 5 -c 1 -o gpurun_out/prof_spmv_fp32 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-cusparse > gpurun_out/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv -s 5 -c 1 -o gpurun_out/prof_spmv_fp16 python bench.py --steps 10 --warmup 3 --dtype fp16 --no-cpu-baseline --no-cusparse >> gpurun_out/ncu_full.log 2>&1
echo done
