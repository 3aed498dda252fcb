#!/bin/bash
# gpu_res3.sh "libs" "workload:hybrid ...": per-library kernel ms + a launch list of the SpMV kernels (first lib)
mkdir -p gpurun_out
bash tools/gpu_res.sh "$1" "$2"
set -- $1
for w in rmat22:2 powerlaw1m:2; do
  wl=${w%%:*}; hy=${w##*:}
  SPADEN_LIB=$PWD/exp/libspaden_$1.so timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__throughput.avg.pct_of_peak_sustained_active --clock-control none -k regex:"k_spmv|k_residual|k_res_chunks|k_res_fixup" -c 12 --csv --log-file gpurun_out/launch3_${wl}_$hy.csv python bench.py --workload $wl --hybrid $hy --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > /dev/null 2>&1
done
