#!/bin/bash
# which build introduced the intermittent dataflow parity failure: 5 repeats of the dataflow tests per build
mkdir -p gpurun_out
cp paper_conf_micro_khorasanieas18_b200/libvpps.so ab/cur.so
: > gpurun_out/flaky2.txt
for so in A C D3 F; do
  cp ab/$so.so paper_conf_micro_khorasanieas18_b200/libvpps.so
  for i in 1 2 3 4 5; do
    echo "$so $(timeout 300 python -m pytest tests -m gpu -q -k 'binary_target_dataflow or dataflow_epochs or dataflow_groups_hidden or dataflow_batch' 2>&1 | grep -E 'passed|failed' | tail -1)" >> gpurun_out/flaky2.txt
  done
done
cp ab/cur.so paper_conf_micro_khorasanieas18_b200/libvpps.so
cat gpurun_out/flaky2.txt
