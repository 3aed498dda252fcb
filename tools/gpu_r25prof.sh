#!/bin/bash
# DRAM / L2 metrics of the rmat25 hybrid kernels (one SpMV)
mkdir -p gpurun_out
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__t_sector_hit_rate.pct,lts__t_tag_requests.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:"k_spmv|k_residual|k_res_chunks|k_res_fixup" -c 6 --csv --log-file gpurun_out/launch_rmat25_2.csv python bench.py --workload rmat25 --hybrid 2 --steps 3 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" > /dev/null 2>&1
python tools/launch_table.py gpurun_out/launch_rmat25_2.csv 2>/dev/null | head -8
