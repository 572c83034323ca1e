#!/bin/bash
# final round-2 evidence with the default launch (vpps_df cooperative, not a programmatic dependent):
# stress of the dataflow selection, two full GPU suites, then the evidence suite and the config sweep
mkdir -p gpurun_out
: > gpurun_out/stress_r2e.txt
f=0
for i in $(seq 1 16); do
  timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/st_tmp.txt 2>&1 || { f=$((f+1)); grep -E "^FAILED" gpurun_out/st_tmp.txt | head -2 >> gpurun_out/stress_r2e.txt; }
done
echo "dataflow selection: failed_runs=$f of 16" >> gpurun_out/stress_r2e.txt
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/tests2_r2e.txt
bash tools/gpu_final.sh r2e
cat gpurun_out/stress_r2e.txt gpurun_out/tests2_r2e.txt gpurun_out/tests_r2e.txt
