#!/bin/bash
# source-level ncu capture of the tiled SpMV (fp32 + fp16, fem1p5m) and a short bench line
mkdir -p gpurun_out/prof
TAG=${TAG:-cur}
timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --spmm "" > gpurun_out/prof/bench_${TAG}.json 2> gpurun_out/prof/bench_${TAG}.err
for dt in fp32 fp16; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o gpurun_out/prof/${TAG}_${dt} python bench.py --steps 10 --warmup 3 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/prof/ncu_${TAG}_${dt}.log 2>&1
done
echo done
