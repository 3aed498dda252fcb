#!/bin/bash
# small / other matrices: kernel ms per env setting (WL workloads), fp32
O=gpurun_out/small; mkdir -p $O; : > $O/summary.txt
for wl in ${WL:-fem62k}; do
for e in ${ENVS:-"SPADEN_STREAM=0" "SPADEN_STREAM_CFG=4" "SPADEN_STREAM_CFG=4 SPADEN_STREAM_CHUNK=64" "SPADEN_STREAM_CFG=1 SPADEN_STREAM_CHUNK=64"}; do
  env $e timeout 300 python bench.py --workload $wl --steps 300 --warmup 10 --dtype ${DT:-fp32} --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > $O/b.json 2> $O/b.err
  python -c "import json; d=json.load(open('$O/b.json')); print('$wl', '[$e]', round(d['roofline']['kernel_ms']*1000,2), 'us', round(d['roofline']['frac'],3))" >> $O/summary.txt 2>&1 || tail -3 $O/b.err >> $O/summary.txt
done; done
cat $O/summary.txt
