#!/bin/bash
# gradient-GEMM items with operands in two cp.async groups (J) against F
mkdir -p gpurun_out
cp ab/J.so paper_conf_micro_khorasanieas18_b200/libvpps.so
timeout 400 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target_config or binary or sgd" 2>&1 | tail -3 > gpurun_out/tests_dw2s.txt
cat gpurun_out/tests_dw2s.txt
bash tools/ab.sh dw2s 3 F:F.so J:J.so
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_dw2s.txt 2>&1
cat gpurun_out/ab_dw2s.txt; sed -n 5,20p gpurun_out/trace_dw2s.txt
