#!/bin/bash
mkdir -p gpurun_out
: > gpurun_out/flaky10.txt
for v in "base:" "dfnopdl:VPPS_DF_NOPDL=1" "dwnopdl:VPPS_DW_NOPDL=1" "coop:VPPS_DF_COOP=1" "base2:"; do
  IFS=: read -r name env <<< "$v"
  ( [ -n "$env" ] && export $env; timeout 900 python tools/flaky_epochs.py 20 2 > gpurun_out/fl10_$name.txt 2>&1 )
  echo "$name $(tail -1 gpurun_out/fl10_$name.txt)" >> gpurun_out/flaky10.txt
  grep "^it" gpurun_out/fl10_$name.txt | head -3 >> gpurun_out/flaky10.txt
done
cat gpurun_out/flaky10.txt
