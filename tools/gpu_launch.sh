#!/bin/bash
# gpu_launch.sh "workload:hybrid ...": ncu launch list (time, DRAM, L2) of the SpMV kernels of each workload
mkdir -p gpurun_out
for w in $1; do
  wl=${w%%:*}; hy=${w##*:}
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__throughput.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:"k_spmv|k_residual|k_res_chunks|k_res_fixup|k_scale" -c 12 --csv --log-file gpurun_out/launch_${wl}_$hy.csv python bench.py --workload $wl --hybrid $hy --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > /dev/null 2>&1
  python tools/launch_table.py gpurun_out/launch_${wl}_$hy.csv | head -8
done
