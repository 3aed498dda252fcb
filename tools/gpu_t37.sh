mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_multi_gpu.py tests/test_gpu_parity.py -k "multi_gpu or symmetric or spmm_tc or two_ranks" -q -x > gpurun_out/t37.log 2>&1; echo rc=$? >> gpurun_out/t37.log
timeout 600 python bench.py --dtype fp16 --steps 50 --warmup 5 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/t37_bench.json 2> gpurun_out/t37_bench.err
