#!/bin/bash
mkdir -p gpurun_out
VPPS_PARITY_STATS=gpurun_out/parity_stats.jsonl timeout 1800 python -m pytest tests -m gpu -q 2>&1 | tail -15 > gpurun_out/tests_r2i.txt
timeout 1500 python tools/config_sweep.py --out gpurun_out/sweep_r2i.jsonl > gpurun_out/sweep_r2i.txt 2>&1
echo done
