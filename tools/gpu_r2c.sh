#!/bin/bash
# gpu tests (all), level-path sweep with the hand-written GEMM, bench
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -25 > gpurun_out/tests_r2c.txt
timeout 900 python tools/config_sweep.py --only "level path" --out gpurun_out/sweep_r2c.jsonl > gpurun_out/sweep_r2c.txt 2>&1
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_r2c.json 2> gpurun_out/bench_r2c.err
echo done
