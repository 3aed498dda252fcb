#!/bin/bash
# separate partial ring configs: tile-config parity test, then kernel us per SPADEN_TILE_CFG (fem1p5m fp32/fp16)
O=gpurun_out/sep; mkdir -p $O; : > $O/summary.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x --timeout 600 -k "every_tile_config or partition_invariance_across or deterministic_and_partition or fem1p5m_full" > $O/pytest.log 2>&1; tail -2 $O/pytest.log >> $O/summary.txt
for rep in 1 2; do for dt in fp32 fp16; do for c in ${CFGS:-15 20 21 22 23}; do
  SPADEN_TILE_CFG=$c timeout 300 python bench.py --steps 500 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > $O/b.json 2> $O/b.err
  python -c "import json; d=json.load(open('$O/b.json')); print('$dt cfg$c', round(d['roofline']['kernel_ms']*1000,2), 'us', round(d['roofline']['frac'],3))" >> $O/summary.txt 2>&1 || tail -2 $O/b.err >> $O/summary.txt
done; done; done
for t in 8 12; do
  timeout 900 python bench.py --workload rmat22 --reorder degree --hybrid $t --steps 300 --warmup 5 --spmm "" --spmm-tc "" --no-variants --no-cpu-baseline --no-cusparse > $O/r.json 2> $O/r.err
  python -c "import json; d=json.load(open('$O/r.json')); print('rmat22 reorder t=$t', round(d['roofline']['kernel_ms'],4), 'ms', round(d['roofline']['frac'],3))" >> $O/summary.txt 2>&1 || tail -2 $O/r.err >> $O/summary.txt
done
cat $O/summary.txt
