#!/bin/bash
# small INT_B batches in every warp without a CTA barrier (G) against F
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target_config or binary" 2>&1 | tail -3 > gpurun_out/tests_wbwd.txt
cat gpurun_out/tests_wbwd.txt
bash tools/ab.sh wbwd 3 F:F.so G:G.so
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_wbwd.txt 2>&1
cat gpurun_out/ab_wbwd.txt
