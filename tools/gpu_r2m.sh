#!/bin/bash
# vpps_df launched without the cooperative attribute (F, default) against the cooperative launch (F + VPPS_DF_COOP=1)
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target_config" 2>&1 | tail -3 > gpurun_out/tests_nocoop.txt
bash tools/ab.sh nocoop 3 coop:F.so:VPPS_DF_COOP=1 free:F.so
timeout 120 python tools/kernel_times.py > gpurun_out/ktimes_nocoop.txt 2>&1
cat gpurun_out/tests_nocoop.txt gpurun_out/ab_nocoop.txt; tail -8 gpurun_out/ktimes_nocoop.txt
