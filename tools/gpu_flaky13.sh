#!/bin/bash
# residual intermittent failure: default launch vs the gradient GEMM also launched normally, 32 runs each
mkdir -p gpurun_out
: > gpurun_out/flaky13.txt
for v in "default:" "dwnopdl:VPPS_DW_NOPDL=1"; do
  IFS=: read -r name env <<< "$v"
  f=0
  for i in $(seq 1 32); do
    ( [ -n "$env" ] && export $env; timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/fl13_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/fl13_tmp.txt | head -4 >> gpurun_out/flaky13.txt; }
  done
  echo "$name failed_runs=$f of 32" >> gpurun_out/flaky13.txt
done
cat gpurun_out/flaky13.txt
