#!/bin/bash
# LEAF_B after the main loop, every leaf's polls in flight at once (L) against F; checked build on the tests
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target_config or binary or sgd" 2>&1 | tail -3 > gpurun_out/tests_leafb.txt
cat gpurun_out/tests_leafb.txt
bash tools/gpu_checked.sh leafb | tail -3
bash tools/ab.sh leafb 3 F:F.so L:L.so
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_leafb.txt 2>&1
cat gpurun_out/ab_leafb.txt; sed -n 1,4p gpurun_out/trace_leafb.txt
