#!/bin/bash
# which pass of the epochs test fails with the programmatic gradient GEMM (VPPS_DW_PDL=1)
mkdir -p gpurun_out
: > gpurun_out/flaky18.txt
f=0
for i in $(seq 1 36); do
  ( export VPPS_DW_PDL=1; timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch' > gpurun_out/fl18_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/fl18_tmp.txt | head -3 >> gpurun_out/flaky18.txt; }
done
echo "VPPS_DW_PDL=1 failed_runs=$f of 36" >> gpurun_out/flaky18.txt
cat gpurun_out/flaky18.txt
