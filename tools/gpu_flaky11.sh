#!/bin/bash
# no programmatic dependent launches on the dataflow path: stress (20 runs of the dataflow selection) + cost
mkdir -p gpurun_out
: > gpurun_out/flaky11.txt
for v in "nopdl:VPPS_DF_NOPDL=1,VPPS_DW_NOPDL=1" "nopdl_coop:VPPS_DF_NOPDL=1,VPPS_DW_NOPDL=1,VPPS_DF_COOP=1"; do
  IFS=: read -r name env <<< "$v"
  f=0
  for i in $(seq 1 20); do
    ( export $(echo $env | tr ',' ' '); timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch or fused_sgd or sgd_step' > gpurun_out/fl11_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^FAILED" gpurun_out/fl11_tmp.txt | head -2 >> gpurun_out/flaky11.txt; }
  done
  echo "$name failed_runs=$f of 20" >> gpurun_out/flaky11.txt
done
bash tools/ab.sh pdl 2 pdl:N.so nopdl:N.so:VPPS_DF_NOPDL=1,VPPS_DW_NOPDL=1 nopdl_coop:N.so:VPPS_DF_NOPDL=1,VPPS_DW_NOPDL=1,VPPS_DF_COOP=1
cat gpurun_out/flaky11.txt gpurun_out/ab_pdl.txt
