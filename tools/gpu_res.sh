#!/bin/bash
# gpu_res.sh "libs" "workload:hybrid ...": kernel ms of the hybrid path per library variant
mkdir -p gpurun_out
: > gpurun_out/res.txt
for w in $2; do for v in $1; do
  wl=${w%%:*}; hy=${w##*:}
  SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 600 python bench.py --workload $wl --hybrid $hy --steps 200 --warmup 5 --no-cpu-baseline --no-variants --spmm "" > gpurun_out/res_${v}_$wl.json 2> gpurun_out/res_${v}_$wl.err
  python -c "import json; d=json.load(open('gpurun_out/res_${v}_$wl.json')); print('$v $w', round(d['roofline']['kernel_ms'],4), 'cusparse', round(d.get('cusparse_csr',{}).get('ms',0),4))" >> gpurun_out/res.txt 2>&1
done; done
cat gpurun_out/res.txt
