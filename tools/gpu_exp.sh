#!/bin/bash
# gpu_exp.sh "v1 v2 ..." [extra bench args]: kernel_ms of exp/libspaden_<v>.so variants (fp32, fp16), 2 passes
mkdir -p gpurun_out
: > gpurun_out/exp.txt
for pass in 1 2; do for v in $1; do for dt in fp32 fp16; do
  SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 600 python bench.py --steps 1000 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" $2 > gpurun_out/exp_${v}_$dt.json 2> gpurun_out/exp_${v}_$dt.err
  python -c "import json; d=json.load(open('gpurun_out/exp_${v}_$dt.json')); print('$v $dt', round(d['roofline']['kernel_ms'],5), round(d['ms_per_step'],5))" >> gpurun_out/exp.txt 2>&1
done; done; done
cat gpurun_out/exp.txt
