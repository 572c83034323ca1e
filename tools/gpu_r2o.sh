#!/bin/bash
# measurement only: gradient-GEMM partial tiles as plain stores (wrong sums) vs red.global.add — is the dW
# tail bound by the L2 reductions?
mkdir -p gpurun_out
bash tools/ab.sh dwstore 2 F:F.so Hst:Hst.so
cp ab/Hst.so paper_conf_micro_khorasanieas18_b200/libvpps.so
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_dwstore.txt 2>&1
cp ab/F.so paper_conf_micro_khorasanieas18_b200/libvpps.so
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_dwred.txt 2>&1
cat gpurun_out/ab_dwstore.txt; sed -n 5,20p gpurun_out/trace_dwstore.txt; sed -n 5,20p gpurun_out/trace_dwred.txt
