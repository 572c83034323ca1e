#!/bin/bash
# every load of the programmatic-dependent kernels through L2 (N): 20 runs of the dataflow selection
mkdir -p gpurun_out
: > gpurun_out/flaky8.txt
f=0
for i in $(seq 1 20); do
  timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/fl8_tmp.txt 2>&1 || { f=$((f+1)); grep -E "^FAILED|Error" gpurun_out/fl8_tmp.txt | head -2 >> gpurun_out/flaky8.txt; }
done
echo "N failed_runs=$f of 20" >> gpurun_out/flaky8.txt
bash tools/ab.sh ldcg 2 F:F.so N:N.so
cat gpurun_out/flaky8.txt gpurun_out/ab_ldcg.txt
