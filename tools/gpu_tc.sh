#!/bin/bash
# tensor-core SpMM: bench numbers at K = 64, 128, 256 + an ncu capture of the kernel
mkdir -p gpurun_out/tc
timeout 900 python bench.py --dtype fp16 --steps 200 --warmup 5 --no-cpu-baseline --no-cusparse --no-variants --spmm "4" --spmm-tc 64,128,256 > gpurun_out/tc/bench.json 2> gpurun_out/tc/bench.err
python -c "import json; d=json.load(open('gpurun_out/tc/bench.json')); print(json.dumps(d['spmm_tc'], indent=1)); print(d['spmm'])"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmm_tc -s 2 -c 1 -o gpurun_out/tc/prof python bench.py --dtype fp16 --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc 128 > gpurun_out/tc/ncu.log 2>&1
echo ncu rc=$?
