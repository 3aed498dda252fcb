#!/bin/bash
# reordering (NEXT-1): GPU tests, then hybrid-auto bench lines with / without --reorder degree
O=gpurun_out/reord; mkdir -p $O; : > $O/summary.txt
timeout 900 python -m pytest tests/test_gpu_reorder.py -q --timeout 600 > $O/pytest.log 2>&1; tail -2 $O/pytest.log >> $O/summary.txt
for wl in ${WL:-powerlaw1m rmat22 rmat25}; do for r in none degree; do
  st=500; [ $wl = rmat25 ] && st=20
  timeout 900 python bench.py --workload $wl --reorder $r --steps $st --warmup 5 --spmm "" --spmm-tc "" --no-variants --cpu-seconds 4 ${ARGS} > $O/b_${wl}_$r.json 2> $O/b_${wl}_$r.err
  python -c "
import json; d=json.load(open('$O/b_${wl}_$r.json'))
c=d['config']; cu=d.get('cusparse_csr') or {}
print('$wl $r', 'ms', round(d['ms_per_step'],4), 'kernel', round(d['roofline']['kernel_ms'],4), 'GF', round(d['value'],1), 'Bnnz', c.get('Bnnz_rank0'), 'fill', round(c.get('fill_rank0',0),2), 't', c.get('hybrid_residual_max_popc'), 'res_nnz', c.get('residual_nnz_rank0'), 'cusparse', cu.get('ms', cu.get('error')), 'speedup', cu.get('speedup_spaden_vs_cusparse'), 'reorder_s', (c.get('reorder') or {}).get('seconds') if isinstance(c.get('reorder'), dict) else None)
" >> $O/summary.txt 2>&1 || tail -3 $O/b_${wl}_$r.err >> $O/summary.txt
done; done
cat $O/summary.txt
