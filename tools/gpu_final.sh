#!/bin/bash
# end-of-round evidence: GPU suite, bench, launch list, ncu captures, DRAM in pipeline, df trace, kernel
# times (tools/run_suite.sh), then the config sweep
TAG=${1:-r2b}
mkdir -p gpurun_out
bash tools/run_suite.sh $TAG
# (compute-sanitizer is closed on the GPU pool from this session on: runs under it had left GPUs needing a
#  reset; the r2b / r2c sanitizer records cover the earlier kernels)
timeout 900 python tools/config_sweep.py --out gpurun_out/sweep_$TAG.jsonl > /dev/null 2> gpurun_out/sweep_$TAG.err
echo done
