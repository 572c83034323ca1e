#!/bin/bash
# the epochs test 20x per launch variant
mkdir -p gpurun_out
: > gpurun_out/flaky7.txt
run() { # name so env
  cp ab/$2.so paper_conf_micro_khorasanieas18_b200/libvpps.so
  local f=0
  for i in $(seq 1 20); do
    ( [ -n "$3" ] && export $(echo $3 | tr ',' ' '); timeout 120 python -m pytest tests -m gpu -q -x -k 'dataflow_epochs' > gpurun_out/fl7_tmp.txt 2>&1 ) || f=$((f+1))
  done
  echo "$1 failed_runs=$f of 20" >> gpurun_out/flaky7.txt
}
run M M ""
run M_dfnopdl M VPPS_DF_NOPDL=1
run M_dwnopdl M VPPS_DW_NOPDL=1
run M_both M VPPS_DF_NOPDL=1,VPPS_DW_NOPDL=1
run M_coop M VPPS_DF_COOP=1
cp ab/M.so paper_conf_micro_khorasanieas18_b200/libvpps.so
cat gpurun_out/flaky7.txt
