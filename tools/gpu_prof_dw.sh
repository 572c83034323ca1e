#!/bin/bash
mkdir -p gpurun_out
TAG=${1:-x}
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"vpps_dw_tc" -s 4 -c 1 -o gpurun_out/prof_dwtc_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_dwtc_$TAG.log 2>&1
echo done
