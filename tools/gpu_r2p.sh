#!/bin/bash
# two FFMA2 groups (8 nodes) per barrier and cell phase in the forward (I) against F
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target_config or binary" 2>&1 | tail -3 > gpurun_out/tests_fs8.txt
cat gpurun_out/tests_fs8.txt
bash tools/ab.sh fs8 3 F:F.so I:I.so
cat gpurun_out/ab_fs8.txt
