#!/bin/bash
# gpu_rmat25.sh: R-MAT scale-25 PageRank (north_star's scaling config) on one GPU, hybrid t=1/2 and pure
mkdir -p gpurun_out
for hy in ${HYS:-1 2 0}; do
  timeout 1200 python bench.py --workload rmat25 --hybrid $hy --steps 20 --warmup 3 --no-variants --spmm "" > gpurun_out/rmat25_$hy.json 2> gpurun_out/rmat25_$hy.err
  python -c "import json; d=json.load(open('gpurun_out/rmat25_$hy.json')); print('rmat25 t=$hy', round(d['roofline']['kernel_ms'],3), 'cusparse', round(d.get('cusparse_csr',{}).get('ms',0),3), d['bytes_per_nnz'])" >> gpurun_out/rmat25.txt 2>&1
done
cat gpurun_out/rmat25.txt
