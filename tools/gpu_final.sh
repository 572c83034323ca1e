#!/bin/bash
# end-of-round evidence: GPU suite, bench, launch list, ncu captures, DRAM in pipeline, df trace, kernel
# times (tools/run_suite.sh), then compute-sanitizer on the changed device paths and the config sweep
TAG=${1:-r2b}
mkdir -p gpurun_out
bash tools/run_suite.sh $TAG
: > gpurun_out/sanitizer_$TAG.txt
for p in dataflow dataflow128 levelgemm chain; do
  for t in memcheck racecheck; do
    echo "== $t $p" >> gpurun_out/sanitizer_$TAG.txt
    timeout 900 compute-sanitizer --tool $t python tools/sanitize_pass.py $p >> gpurun_out/sanitizer_$TAG.txt 2>&1
    echo "rc=$?" >> gpurun_out/sanitizer_$TAG.txt
  done
done
timeout 900 python tools/config_sweep.py --out gpurun_out/sweep_$TAG.jsonl > /dev/null 2> gpurun_out/sweep_$TAG.err
echo done
