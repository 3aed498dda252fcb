#!/bin/bash
# round-end style check: smoke, full GPU suite, default bench (+clocks), launch list, ncu full of the SpMV
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/clocks.csv &
SMI=$!
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
kill $SMI
timeout 600 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 30 -c 60 --csv --log-file gpurun_out/launches_fp32.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-variants > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o gpurun_out/prof_final_fp32 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants > gpurun_out/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o gpurun_out/prof_final_fp16 python bench.py --steps 10 --warmup 3 --dtype fp16 --no-cpu-baseline --no-cusparse --no-variants >> gpurun_out/ncu_full.log 2>&1
echo done
