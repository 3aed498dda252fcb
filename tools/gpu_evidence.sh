#!/bin/bash
# gpu_evidence.sh: bench lines of the non-default workloads (profiles/r01_bench_*), residual ncu capture
mkdir -p gpurun_out/ev
for w in ${WLS:-fem62k:0 powerlaw1m:0 powerlaw1m:4 rmat22:0 rmat22:3 fem1p5m:0}; do
  wl=${w%%:*}; hy=${w##*:}
  dt=fp32
  timeout 900 python bench.py --workload $wl --hybrid $hy --steps 500 --warmup 10 --spmm "" --cpu-seconds 8 > gpurun_out/ev/r01_bench_${wl}_$hy.json 2> gpurun_out/ev/r01_bench_${wl}_$hy.err
done
timeout 900 python bench.py --workload fem1p5m --dtype fp16 --steps 500 --warmup 10 --spmm "" --cpu-seconds 8 > gpurun_out/ev/r01_bench_fem1p5m_fp16.json 2> gpurun_out/ev/r01_bench_fem1p5m_fp16.err
[ -n "$NONCU" ] || timeout 900 ncu --set full --clock-control none --import-source on -k regex:residual_binned -s 3 -c 1 -o gpurun_out/ev/prof_res_rmat22_t3 python bench.py --workload rmat22 --hybrid 3 --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > /dev/null 2>&1
[ -n "$NONCU" ] || bash tools/gpu_launch.sh "rmat22:3 powerlaw1m:4" > gpurun_out/ev/launch_tables.txt 2>&1
for f in gpurun_out/ev/r01_bench_*.json; do python -c "import json,sys; d=json.load(open('$f')); print('$f', d['config']['workload'], d['dtype'], round(d['roofline']['kernel_ms'],4), round(d['roofline']['frac'],3), 'cusparse', round(d.get('cusparse_csr',{}).get('ms',0),4))" ; done
