#!/bin/bash
# H = 128 dataflow groups: parity + throughput against the level / grid paths
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "hidden_128 or dataflow_groups or target_dataflow" 2>&1 | tail -15 > gpurun_out/tests_h128.txt
timeout 600 python tools/config_sweep.py --only H128 > gpurun_out/sweep_h128.jsonl 2> gpurun_out/sweep_h128.err
echo done
