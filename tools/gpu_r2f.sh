#!/bin/bash
# final launch configuration (no programmatic launches on the dataflow path): stress, suite, evidence
mkdir -p gpurun_out
: > gpurun_out/stress_r2f.txt
f=0
for i in $(seq 1 24); do
  timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/stf_tmp.txt 2>&1 || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/stf_tmp.txt | head -4 >> gpurun_out/stress_r2f.txt; }
done
echo "dataflow selection: failed_runs=$f of 24" >> gpurun_out/stress_r2f.txt
bash tools/ab.sh final 2 T:T.so T_dwpdl:T.so:VPPS_DW_PDL=1
bash tools/run_suite.sh r2f
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2f.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_r2f.txt
cat gpurun_out/stress_r2f.txt gpurun_out/ab_final.txt gpurun_out/tests_r2f.txt gpurun_out/smoke_r2f.txt
