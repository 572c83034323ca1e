#!/bin/bash
# gradient GEMM at 4 CTAs per SM (64-node items, 64-row leaf-dX chunks; K) against 3 (F)
mkdir -p gpurun_out
cp ab/K.so paper_conf_micro_khorasanieas18_b200/libvpps.so
timeout 400 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target_config or binary or sgd" 2>&1 | tail -3 > gpurun_out/tests_dw4.txt
cat gpurun_out/tests_dw4.txt
bash tools/ab.sh dw4 3 F:F.so K:K.so
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_dw4.txt 2>&1
cp ab/F.so paper_conf_micro_khorasanieas18_b200/libvpps.so
cat gpurun_out/ab_dw4.txt; sed -n 5,20p gpurun_out/trace_dw4.txt
