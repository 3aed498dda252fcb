#!/bin/bash
# gpu_pdl.sh "workload:hybrid ...": kernel ms with programmatic dependent launch on / off (SPADEN_PDL=0)
mkdir -p gpurun_out
: > gpurun_out/pdl.txt
[ -n "$NOTEST" ] || { timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_pdl.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_pdl.log; }
tail -2 gpurun_out/pytest_pdl.log >> gpurun_out/pdl.txt
for rep in 1 2; do for w in $1; do for p in 1 0; do
  wl=${w%%:*}; hy=${w##*:}
  SPADEN_PDL=$p timeout 600 python bench.py --workload $wl --hybrid $hy --steps ${STEPS:-300} --warmup 5 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/pdl_$p.json 2> gpurun_out/pdl_$p.err
  python -c "import json; d=json.load(open('gpurun_out/pdl_$p.json')); print('pdl=$p $w', round(d['roofline']['kernel_ms'],4))" >> gpurun_out/pdl.txt 2>&1
done; done; done
cat gpurun_out/pdl.txt
