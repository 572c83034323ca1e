#!/bin/bash
mkdir -p gpurun_out
timeout 900 python tools/flaky_epochs.py 8 1 > gpurun_out/flaky9.txt 2>&1
VPPS_DF_NOPDL=1 VPPS_DW_NOPDL=1 VPPS_DF_COOP=1 timeout 900 python tools/flaky_epochs.py 8 1 > gpurun_out/flaky9b.txt 2>&1
tail -20 gpurun_out/flaky9.txt; echo ---; tail -8 gpurun_out/flaky9b.txt
