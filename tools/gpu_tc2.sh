#!/bin/bash
# tensor-core SpMM: parity tests + bench timing (K = 64, 128)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -k "spmm_tc" -q -x > gpurun_out/tc2.log 2>&1; echo rc=$? >> gpurun_out/tc2.log
timeout 600 python bench.py --dtype fp16 --steps 50 --warmup 5 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/tc2_bench.json 2> gpurun_out/tc2_bench.err
python -c "import json; d=json.loads(open('gpurun_out/tc2_bench.json').read().strip().splitlines()[-1]); print({k: (round(v['ms'],4), round(v['gflops'])) for k, v in d['spmm_tc'].items()})" >> gpurun_out/tc2.log 2>&1
SPADEN_LIB=$PWD/exp/libspaden_tctrace.so PYTHONPATH=$PWD timeout 300 python tools/tc_trace.py 128 > gpurun_out/tctrace.txt 2>&1
