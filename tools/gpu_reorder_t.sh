#!/bin/bash
# hybrid threshold sweep with --reorder degree: kernel ms per (workload, t)
O=gpurun_out/reordt; mkdir -p $O; : > $O/summary.txt
for wl in ${WL:-rmat22 rmat25}; do for t in ${TS:-1 2 3 4 6}; do
  st=300; [ $wl = rmat25 ] && st=20
  timeout 900 python bench.py --workload $wl --reorder ${REORDER:-degree} --hybrid $t --steps $st --warmup 5 --spmm "" --spmm-tc "" --no-variants --no-cpu-baseline --no-cusparse > $O/b.json 2> $O/b.err
  python -c "
import json; d=json.load(open('$O/b.json')); c=d['config']
print('$wl t=$t', 'kernel_ms', round(d['roofline']['kernel_ms'],4), 'frac', round(d['roofline']['frac'],3), 'res_nnz', c.get('residual_nnz_rank0'), 'parts', c.get('residual_parts'))
" >> $O/summary.txt 2>&1 || tail -3 $O/b.err >> $O/summary.txt
done; done
cat $O/summary.txt
