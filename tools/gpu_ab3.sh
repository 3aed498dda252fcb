#!/bin/bash
# gpu_ab3.sh: kernel ms per experiment library (LIBS), workload (WL) and dtype (DTS), twice, interleaved
O=gpurun_out/ab3; mkdir -p $O; : > $O/summary.txt
for rep in 1 2; do for wl in ${WL:-fem1p5m}; do for dt in ${DTS:-fp32 fp16}; do for v in ${LIBS}; do
  SPADEN_LIB=$PWD/exp/libspaden_$v.so timeout ${BENCH_TIMEOUT:-180} python bench.py --workload $wl --dtype $dt --steps ${STEPS:-500} --warmup 10 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" ${ARGS} > $O/b.json 2> $O/b.err
  python -c "import json; d=json.load(open('$O/b.json')); print('$v $wl $dt', round(d['roofline']['kernel_ms']*1000,2), 'us', round(d['roofline']['frac'],3))" >> $O/summary.txt 2>&1 || tail -2 $O/b.err >> $O/summary.txt
done; done; done; done
if [ -n "$TESTLIB" ]; then SPADEN_LIB=$PWD/exp/libspaden_$TESTLIB.so timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $O/pytest.log 2>&1; tail -2 $O/pytest.log >> $O/summary.txt; fi
cat $O/summary.txt
