#!/bin/bash
# tensor-core SpMM: K=64/128 ms per experiment library (LIBS), twice
O=gpurun_out/tcab; mkdir -p $O; : > $O/summary.txt
for rep in 1 2; do for v in ${LIBS}; do
  SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout 180 python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc 64,128 > $O/b.json 2> $O/b.err
  python -c "import json; d=json.load(open('$O/b.json')); t=d['spmm_tc']; print('$v', 'K64', round(t['64']['ms'],4), 'K128', round(t['128']['ms'],4))" >> $O/summary.txt 2>&1 || tail -2 $O/b.err >> $O/summary.txt
done; done
if [ -n "$TESTLIB" ]; then SPADEN_LIB=$PWD/exp/libspaden_$TESTLIB.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "spmm_tc" > $O/pytest.log 2>&1; tail -2 $O/pytest.log >> $O/summary.txt; fi
cat $O/summary.txt
