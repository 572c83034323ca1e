#!/bin/bash
# intermittent corruption: 15 pytest runs of the dataflow selection per variant
mkdir -p gpurun_out
: > gpurun_out/flaky5.txt
run() { # name so env
  cp ab/$2.so paper_conf_micro_khorasanieas18_b200/libvpps.so
  local f=0
  for i in $(seq 1 15); do
    ( [ -n "$3" ] && export $(echo $3 | tr ',' ' '); timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch' > gpurun_out/fl5_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^FAILED|Error" gpurun_out/fl5_tmp.txt | head -2 >> gpurun_out/flaky5.txt; }
  done
  echo "$1 failed_runs=$f of 15" >> gpurun_out/flaky5.txt
}
run F F ""
run F_dwnopdl F VPPS_DW_NOPDL=1
run F_nopdl_all F VPPS_DW_NOPDL=1,VPPS_DF_NOPDL=1,VPPS_DF_COOP=1
run A A ""
cp ab/F.so paper_conf_micro_khorasanieas18_b200/libvpps.so
cat gpurun_out/flaky5.txt
