#!/bin/bash
# release pattern of vpps_df's done counters (barrier, then fence + release add by thread 0), with the
# gradient GEMM programmatic again (VPPS_DW_PDL=1): 32 stress runs
mkdir -p gpurun_out
: > gpurun_out/flaky16.txt
f=0
for i in $(seq 1 32); do
  ( export VPPS_DW_PDL=1; timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/fl16_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/fl16_tmp.txt | head -3 >> gpurun_out/flaky16.txt; }
done
echo "U + VPPS_DW_PDL=1 failed_runs=$f of 32" >> gpurun_out/flaky16.txt
bash tools/ab.sh relpat 2 T:T.so U:U.so U_pdl:U.so:VPPS_DW_PDL=1
cat gpurun_out/flaky16.txt gpurun_out/ab_relpat.txt
