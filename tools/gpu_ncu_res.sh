#!/bin/bash
mkdir -p gpurun_out
for w in rmat22:2 powerlaw1m:1; do
  wl=${w%%:*}; hy=${w##*:}
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,lts__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__throughput.avg.pct_of_peak_sustained_active --clock-control none -k regex:"spmv|res|fixup|chunk" -s 4 -c 12 --csv --log-file gpurun_out/launch_${wl}_$hy.csv python bench.py --workload $wl --hybrid $hy --steps 10 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > /dev/null 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:residual_binned -s 3 -c 1 -o gpurun_out/prof_res_rmat22 python bench.py --workload rmat22 --hybrid 2 --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > /dev/null 2>&1
echo done
