#!/bin/bash
# launch list of the timed region only (NVTX range bench_timed_region), fem1p5m fp32 and rmat22 hybrid
O=gpurun_out/nvtx; mkdir -p $O
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > $O/bench.json 2> $O/bench.err; tail -c 300 $O/bench.json
timeout 600 ncu --nvtx --nvtx-include "bench_timed_region/" --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_timed_fem1p5m_fp32.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > /dev/null 2>&1
timeout 600 ncu --nvtx --nvtx-include "bench_timed_region/" --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_timed_rmat22_hybrid.csv python bench.py --workload rmat22 --steps 5 --warmup 3 --no-cpu-baseline --no-cusparse --no-variants --spmm "" --spmm-tc "" > /dev/null 2>&1
ls -la $O
