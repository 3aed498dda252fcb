#!/bin/bash
# gpu_res2.sh "workload:hybrid ...": hybrid residual, binned (default) vs the fixed 16-lane kernel (SPADEN_RES=fixed)
mkdir -p gpurun_out
: > gpurun_out/res2.txt
timeout 900 python -m pytest tests -m gpu -q -x -k "hybrid or residual or random_shapes or spmm_hybrid" > gpurun_out/pytest_res.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_res.log
tail -3 gpurun_out/pytest_res.log >> gpurun_out/res2.txt
for w in $1; do for v in binned fixed; do
  wl=${w%%:*}; hy=${w##*:}
  SPADEN_RES=$v timeout 600 python bench.py --workload $wl --hybrid $hy --steps 200 --warmup 5 --no-cpu-baseline --no-variants --spmm "" > gpurun_out/res2_${v}_${wl}_$hy.json 2> gpurun_out/res2_${v}_${wl}_$hy.err
  python -c "import json; d=json.load(open('gpurun_out/res2_${v}_${wl}_$hy.json')); print('$v $w', round(d['roofline']['kernel_ms'],4), 'cusparse', round(d.get('cusparse_csr',{}).get('ms',0),4))" >> gpurun_out/res2.txt 2>&1
done; done
cat gpurun_out/res2.txt
