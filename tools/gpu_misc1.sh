#!/bin/bash
O=gpurun_out/misc1; mkdir -p $O; : > $O/summary.txt
for p in 0 1; do
  SPADEN_ROT_PASSES=$p timeout 300 python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > $O/b.json 2> $O/b.err
  python -c "import json; d=json.load(open('$O/b.json')); print('passes=$p convert', d['convert']['seconds'], d['convert']['reps_seconds'], 'kernel', d['roofline']['kernel_ms'])" >> $O/summary.txt
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o $O/fem62k python bench.py --workload fem62k --steps 10 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > /dev/null 2>&1
ncu -i $O/fem62k.ncu-rep --page source --csv --print-source sass > $O/src_fem62k.csv 2>/dev/null
ncu -i $O/fem62k.ncu-rep --page raw --csv > $O/raw_fem62k.csv 2>/dev/null
python tools/ncu_summary.py $O/fem62k.ncu-rep >> $O/summary.txt 2>&1
rm -f $O/fem62k.ncu-rep
cat $O/summary.txt
