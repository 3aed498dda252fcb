#!/bin/bash
# rmat25 hybrid t=2 kernel ms vs residual column-part size (SPADEN_XSEG_COLS)
mkdir -p gpurun_out
: > gpurun_out/xseg.txt
for c in ${COLS:-2097152 4194304 8388608 16777216 67108864}; do
  SPADEN_XSEG_COLS=$c timeout 900 python bench.py --workload rmat25 --hybrid 2 --steps 20 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/xseg_$c.json 2> gpurun_out/xseg_$c.err
  python -c "import json; d=json.load(open('gpurun_out/xseg_$c.json')); print('seg_cols $c', round(d['roofline']['kernel_ms'],3))" >> gpurun_out/xseg.txt 2>&1
done
cat gpurun_out/xseg.txt
