#!/bin/bash
# small-matrix tile configs (SPADEN_TILE_CFG) with an experiment library: kernel us, two repetitions
O=gpurun_out/scfg; mkdir -p $O; : > $O/summary.txt
for rep in 1 2; do for wl in ${WL:-fem62k powerlaw1m}; do for c in ${CFGS:-5 3 24 25 26}; do
  SPADEN_LIB=$PWD/exp/libspaden_${LIB:-single}.so SPADEN_TILE_CFG=$c timeout 300 python bench.py --workload $wl --steps 300 --warmup 10 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > $O/b.json 2> $O/b.err
  python -c "import json; d=json.load(open('$O/b.json')); print('$wl cfg$c', round(d['roofline']['kernel_ms']*1000,2), 'us', round(d['roofline']['frac'],3))" >> $O/summary.txt 2>&1 || tail -2 $O/b.err >> $O/summary.txt
done; done; done
cat $O/summary.txt
