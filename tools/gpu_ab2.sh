#!/bin/bash
# gpu_ab2.sh "libs" "workloads": kernel ms per experiment library and workload (fp32), twice, interleaved
mkdir -p gpurun_out
: > gpurun_out/ab.txt
for rep in 1 2; do for wl in $2; do for v in $1; do
  SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 600 python bench.py --workload $wl --steps 500 --warmup 10 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > gpurun_out/ab_${v}_$wl.json 2> gpurun_out/ab_${v}_$wl.err
  python -c "import json; d=json.load(open('gpurun_out/ab_${v}_$wl.json')); print('$v $wl', round(d['roofline']['kernel_ms']*1000,2), 'us')" >> gpurun_out/ab.txt 2>&1
done; done; done
cat gpurun_out/ab.txt
