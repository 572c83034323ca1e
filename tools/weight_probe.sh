#!/bin/bash
# usage: bash tools/weight_probe.sh TAG — DRAM bytes of each kernel for a batch of ONE tree (the smallest
# script: prologue weights dominate), caches flushed before every kernel (ncu default): the weight-traffic
# probe of SURVEY §8(d) against weights-once
TAG=$1
mkdir -p gpurun_out
timeout 300 ncu --cache-control all --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --csv --log-file gpurun_out/wprobe_$TAG.csv python bench.py --batch 1 --steps 4 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
echo done
