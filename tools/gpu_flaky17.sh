#!/bin/bash
# second stress of the release-pattern fix with the programmatic gradient GEMM (40 runs), then the bench
mkdir -p gpurun_out
: > gpurun_out/flaky17.txt
f=0
for i in $(seq 1 40); do
  ( export VPPS_DW_PDL=1; timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/fl17_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/fl17_tmp.txt | head -3 >> gpurun_out/flaky17.txt; }
done
echo "U + VPPS_DW_PDL=1 failed_runs=$f of 40" >> gpurun_out/flaky17.txt
cat gpurun_out/flaky17.txt
