#!/bin/bash
# gpu_ab.sh "libs" [workload]: fem1p5m (default) fp32/fp16 kernel ms per experiment library, twice, interleaved
mkdir -p gpurun_out
wl=${2:-fem1p5m}
: > gpurun_out/ab.txt
for rep in 1 2; do for v in $1; do for dt in fp32 fp16; do
  SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 600 python bench.py --workload $wl --steps 1000 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/ab_${v}_$dt.json 2> gpurun_out/ab_${v}_$dt.err
  python -c "import json; d=json.load(open('gpurun_out/ab_${v}_$dt.json')); print('$v $dt', round(d['roofline']['kernel_ms'],4))" >> gpurun_out/ab.txt 2>&1
done; done; done
cat gpurun_out/ab.txt
