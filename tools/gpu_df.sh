#!/bin/bash
# dataflow-path check: parity tests of the bench's path, bench (no CPU baseline), df trace
TAG=${1:-x}
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target or dp_ or sgd_step" 2>&1 | tail -3 > gpurun_out/tests_$TAG.txt
for i in 1 2; do timeout 300 python bench.py --no-cpu-baseline --steps 200 > gpurun_out/bench_${TAG}_$i.json 2> gpurun_out/bench_${TAG}_$i.err; done
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_$TAG.txt 2>&1
echo done
