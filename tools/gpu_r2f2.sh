#!/bin/bash
# loss by stream-ordered copy on every path (S): stress of the dataflow selection, full suite, A/B against R
mkdir -p gpurun_out
: > gpurun_out/stress_s.txt
f=0
for i in $(seq 1 24); do
  timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step or stale' > gpurun_out/sts_tmp.txt 2>&1 || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/sts_tmp.txt | head -4 >> gpurun_out/stress_s.txt; }
done
echo "S dataflow selection: failed_runs=$f of 24" >> gpurun_out/stress_s.txt
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/tests_s.txt
bash tools/ab.sh lossmc 3 R:R.so S:S.so
cat gpurun_out/stress_s.txt gpurun_out/tests_s.txt gpurun_out/ab_lossmc.txt
