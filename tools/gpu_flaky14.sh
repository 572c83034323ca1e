#!/bin/bash
# loss copied by a stream-ordered memcpy after the gradient GEMM instead of in its tail (VPPS_LOSS_MEMCPY=1)
mkdir -p gpurun_out
: > gpurun_out/flaky14.txt
f=0
for i in $(seq 1 32); do
  ( export VPPS_LOSS_MEMCPY=1; timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/fl14_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/fl14_tmp.txt | head -4 >> gpurun_out/flaky14.txt; }
done
echo "lossmemcpy failed_runs=$f of 32" >> gpurun_out/flaky14.txt
cat gpurun_out/flaky14.txt
