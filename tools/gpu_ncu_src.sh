#!/bin/bash
# ncu --set full (with source counters) of one k_spmv_tiled launch on fem1p5m, fp32 and fp16
# usage: DTS="fp32 fp16" TAG=x bash tools/gpu_ncu_src.sh
O=gpurun_out/ncu_${TAG:-src}; mkdir -p $O
for dt in ${DTS:-fp32 fp16}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-spmv_tiled} -s 5 -c 1 -o $O/spmv_$dt python bench.py --steps 10 --warmup 3 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" ${ARGS} > $O/log_$dt.txt 2>&1
  ncu -i $O/spmv_$dt.ncu-rep --page source --csv --print-source sass > $O/src_$dt.csv 2>/dev/null
  ncu -i $O/spmv_$dt.ncu-rep --page raw --csv > $O/raw_$dt.csv 2>/dev/null
done
ls -la $O
