#!/bin/bash
# gradient GEMM launched programmatically but starting no item before every vpps_df group is done
mkdir -p gpurun_out
: > gpurun_out/flaky15.txt
f=0
for i in $(seq 1 32); do
  ( export VPPS_DW_WAITALL=1; timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/fl15_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/fl15_tmp.txt | head -4 >> gpurun_out/flaky15.txt; }
done
echo "waitall failed_runs=$f of 32" >> gpurun_out/flaky15.txt
bash tools/ab.sh waitall 2 default:R.so waitall:R.so:VPPS_DW_WAITALL=1
cat gpurun_out/flaky15.txt gpurun_out/ab_waitall.txt
