#!/bin/bash
# ncu full capture (source-level) of the dominant kernel and the two GEMMs of the bench step
TAG=${1:-r2p}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"vpps_df" -s 8 -c 1 -o gpurun_out/prof_df_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_df_$TAG.log 2>&1
timeout 300 python tools/df_trace.py --batches > gpurun_out/trace_$TAG.txt 2>&1
echo done
