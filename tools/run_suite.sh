#!/bin/bash
# usage: bash tools/run_suite.sh TAG  — gpu tests, bench, launch list, ncu full capture of the hot kernels,
# dataflow trace, per-kernel times
TAG=$1
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/tests_$TAG.txt; cat gpurun_out/tests_$TAG.txt
timeout 300 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"vpps_df|dw_gemm|leaf_fwd" -s 8 -c 3 -o gpurun_out/prof_$TAG python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_$TAG.log 2>&1
timeout 300 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --csv --log-file gpurun_out/dram_inpipe_$TAG.csv python bench.py --steps 6 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_$TAG.txt 2>&1
timeout 120 python tools/kernel_times.py > gpurun_out/ktimes_$TAG.txt 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_$TAG.txt
echo done
