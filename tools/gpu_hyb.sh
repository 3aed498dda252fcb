#!/bin/bash
# gpu_hyb.sh "workload:hybrid ...": hybrid-path GPU tests + kernel ms per workload
mkdir -p gpurun_out
: > gpurun_out/hyb.txt
timeout 900 python -m pytest tests -m gpu -q -x -k "hybrid or residual or random_shapes or spmm or tile_row_cap or host or graph or long or pagerank or hub or configs" > gpurun_out/pytest_hyb.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_hyb.log
tail -3 gpurun_out/pytest_hyb.log >> gpurun_out/hyb.txt
for w in $1; do
  wl=${w%%:*}; hy=${w##*:}
  timeout 600 python bench.py --workload $wl --hybrid $hy --steps 200 --warmup 5 --no-cpu-baseline --no-variants --spmm "" > gpurun_out/hyb_${wl}_$hy.json 2> gpurun_out/hyb_${wl}_$hy.err
  python -c "import json; d=json.load(open('gpurun_out/hyb_${wl}_$hy.json')); print('$w', round(d['roofline']['kernel_ms'],4), 'cusparse', round(d.get('cusparse_csr',{}).get('ms',0),4))" >> gpurun_out/hyb.txt 2>&1
done
for w in rmat22:2 powerlaw1m:2; do
  wl=${w%%:*}; hy=${w##*:}
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__throughput.avg.pct_of_peak_sustained_active --clock-control none -k regex:"k_spmv|k_residual|k_res_chunks|k_res_fixup|k_scale" -c 12 --csv --log-file gpurun_out/launch_hyb_${wl}_$hy.csv python bench.py --workload $wl --hybrid $hy --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > /dev/null 2>&1
done
cat gpurun_out/hyb.txt
