#!/bin/bash
# record operands of vpps_df through L2 (V1) with the programmatic gradient GEMM: 36 stress runs
mkdir -p gpurun_out
cp ab/V1.so paper_conf_micro_khorasanieas18_b200/libvpps.so
: > gpurun_out/flaky19.txt
f=0
for i in $(seq 1 36); do
  ( export VPPS_DW_PDL=1; timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch' > gpurun_out/fl19_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^E  |^FAILED" gpurun_out/fl19_tmp.txt | head -2 >> gpurun_out/flaky19.txt; }
done
echo "V1 (L2 record loads) + VPPS_DW_PDL=1 failed_runs=$f of 36" >> gpurun_out/flaky19.txt
cat gpurun_out/flaky19.txt
