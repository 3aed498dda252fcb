#!/bin/bash
# round-2 final evidence at HEAD: smoke, GPU tests, bench lines, launch list, ncu summaries, sanitizers
O=gpurun_out/ev3; mkdir -p $O
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench_fem1p5m_fp32.json 2> $O/bench_fem1p5m_fp32.err
timeout 900 python bench.py --dtype fp16 --spmm "" > $O/bench_fem1p5m_fp16.json 2> $O/bench_fem1p5m_fp16.err
timeout 600 python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err
for w in fem62k:0 powerlaw1m:-1 powerlaw1m:0 rmat22:-1 rmat22:0; do
  wl=${w%%:*}; hy=${w##*:}
  timeout 900 python bench.py --workload $wl --hybrid $hy --steps 500 --warmup 10 --spmm "" --spmm-tc "" --cpu-seconds 6 > $O/bench_${wl}_h$hy.json 2> $O/bench_${wl}_h$hy.err
done
timeout 900 python bench.py --workload rmat25 --steps 20 --warmup 3 --spmm "" --spmm-tc "" --no-variants --cpu-seconds 6 > $O/bench_rmat25_h-1.json 2> $O/bench_rmat25_h-1.err
timeout 900 python bench.py --workload rmat25 --reorder degree --steps 20 --warmup 3 --spmm "" --spmm-tc "" --no-variants --cpu-seconds 6 > $O/bench_rmat25_h-1_reorder.json 2> $O/bench_rmat25_h-1_reorder.err
# launch list of the timed step (the SpMV kernel is the only kernel of a fem1p5m step)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"spmv|spmm|spaden|residual|long" -c 60 --csv --log-file $O/launches_fem1p5m_fp32.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > /dev/null 2>&1
for dt in fp32 fp16; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_tiled -s 5 -c 1 -o $O/ncu_spmv_$dt python bench.py --steps 10 --warmup 3 --dtype $dt --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > /dev/null 2>&1
  python tools/ncu_summary.py $O/ncu_spmv_$dt.ncu-rep > $O/ncu_summary_spmv_$dt.txt 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmm_tc -s 2 -c 1 -o $O/ncu_spmm_tc python bench.py --dtype fp16 --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc 128 > /dev/null 2>&1
python tools/ncu_summary.py $O/ncu_spmm_tc.ncu-rep > $O/ncu_summary_spmm_tc.txt 2>&1
timeout 900 ncu --set full --clock-control none -k regex:residual -s 3 -c 1 -o $O/ncu_residual_rmat22 python bench.py --workload rmat22 --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > /dev/null 2>&1
python tools/ncu_summary.py $O/ncu_residual_rmat22.ncu-rep > $O/ncu_summary_residual_rmat22.txt 2>&1
for tool in ${SANITIZERS:-}; do
  timeout 900 compute-sanitizer --tool $tool --target-processes all python tools/sanitize_run.py > $O/sanitizer_$tool.log 2>&1; echo "rc=$?" >> $O/sanitizer_$tool.log
done
rm -f $O/*.ncu-rep.tmp
echo "evidence done"
rm -f $O/*.ncu-rep
