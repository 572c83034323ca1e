#!/bin/bash
mkdir -p gpurun_out
timeout 600 python tools/flaky_diag.py 5 10 > gpurun_out/flaky3.txt 2>&1
cp ab/A.so paper_conf_micro_khorasanieas18_b200/libvpps.so
timeout 600 python tools/flaky_diag.py 5 6 >> gpurun_out/flaky3.txt 2>&1
cat gpurun_out/flaky3.txt
