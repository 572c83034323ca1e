#!/bin/bash
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q 2>&1 | tail -15 > gpurun_out/tests_r2h.txt
timeout 600 python bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench2_r2h.json 2> gpurun_out/bench2_r2h.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/benchref_r2h.json 2>&1
echo done
