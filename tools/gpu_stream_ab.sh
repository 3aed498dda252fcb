#!/bin/bash
# warp-streamed kernel: GPU tests, then fem1p5m kernel ms: CTA-pipeline (SPADEN_STREAM=0) vs stream cfgs
O=gpurun_out/sab; mkdir -p $O; : > $O/summary.txt
if [ -z "$NOTEST" ]; then
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -3 $O/pytest_gpu.log >> $O/summary.txt
fi
for dt in fp32 fp16; do
for e in ${ENVS:-"SPADEN_STREAM=0" "SPADEN_STREAM_CFG=0" "SPADEN_STREAM_CFG=1" "SPADEN_STREAM_CFG=2"}; do
  env $e timeout 300 python bench.py --steps 500 --warmup 10 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" ${ARGS} > $O/b.json 2> $O/b.err
  python -c "import json; d=json.load(open('$O/b.json')); print('$dt', '[$e]', round(d['roofline']['kernel_ms'],4), round(d['roofline']['frac'],3))" >> $O/summary.txt 2>&1 || tail -3 $O/b.err >> $O/summary.txt
done; done
cat $O/summary.txt
