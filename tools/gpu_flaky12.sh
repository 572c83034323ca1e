#!/bin/bash
# programmatic launch of the gradient GEMM only (vpps_df launched after the leaf GEMM completes)
mkdir -p gpurun_out
: > gpurun_out/flaky12.txt
f=0
for i in $(seq 1 24); do
  ( export VPPS_DF_NOPDL=1; timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/fl12_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^FAILED" gpurun_out/fl12_tmp.txt | head -2 >> gpurun_out/flaky12.txt; }
done
echo "dfnopdl failed_runs=$f of 24" >> gpurun_out/flaky12.txt
bash tools/ab.sh pdl2 2 pdl:N.so dfnopdl:N.so:VPPS_DF_NOPDL=1
cat gpurun_out/flaky12.txt gpurun_out/ab_pdl2.txt
