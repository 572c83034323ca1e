#!/bin/bash
# intermittent corruption after routing cross-grid pool reads through L2 (M): 20 pytest runs
mkdir -p gpurun_out
: > gpurun_out/flaky6.txt
run() { # name so env
  cp ab/$2.so paper_conf_micro_khorasanieas18_b200/libvpps.so
  local f=0
  for i in $(seq 1 20); do
    ( [ -n "$3" ] && export $(echo $3 | tr ',' ' '); timeout 300 python -m pytest tests -m gpu -q -x -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch' > gpurun_out/fl6_tmp.txt 2>&1 ) || { f=$((f+1)); grep -E "^FAILED|Error" gpurun_out/fl6_tmp.txt | head -2 >> gpurun_out/flaky6.txt; }
  done
  echo "$1 failed_runs=$f of 20" >> gpurun_out/flaky6.txt
}
run M M ""
cp ab/M.so paper_conf_micro_khorasanieas18_b200/libvpps.so
bash tools/ab.sh l2reads 2 F:F.so M:M.so
cat gpurun_out/flaky6.txt gpurun_out/ab_l2reads.txt
