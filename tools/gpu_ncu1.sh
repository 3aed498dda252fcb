#!/bin/bash
# one ncu --set full capture: CFG=<tile cfg> DT=<fp32|fp16> TAG=<name> [K=<kernel regex>]
mkdir -p gpurun_out/ncu
SPADEN_TILE_CFG=${CFG} timeout 600 ncu --set full --clock-control none --import-source on -k regex:${K:-spmv_wp} -s 5 -c 1 -o gpurun_out/ncu/${TAG} python bench.py --steps 10 --warmup 3 --dtype ${DT:-fp32} --no-cpu-baseline --no-cusparse --no-variants --spmm "" > gpurun_out/ncu/${TAG}.log 2>&1
echo rc=$?
