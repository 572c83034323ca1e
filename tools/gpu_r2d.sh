#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gemm_gpu.py -q -x 2>&1 | tail -25 > gpurun_out/tests_r2d.txt
timeout 900 python -m pytest tests -m gpu -q -x -k "level or tagger or full_size or config5 or gru or rvnn or td" 2>&1 | tail -5 >> gpurun_out/tests_r2d.txt
timeout 900 python tools/config_sweep.py --only "level path" --out gpurun_out/sweep_r2d.jsonl > gpurun_out/sweep_r2d.txt 2>&1
echo done
