#!/bin/bash
# usage: bash tools/quick.sh TAG — dataflow parity tests, bench (no CPU baseline), df trace, kernel times
TAG=$1
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -k "dataflow or fused_sgd or target_config" 2>&1 | tail -3 > gpurun_out/tests_$TAG.txt; cat gpurun_out/tests_$TAG.txt
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json | python -c "import json,sys; d=json.load(sys.stdin); print('value',d['value'],'ms',d['ms_per_step'],'df_ms',d['roofline']['kernel_ms'],'e2e',d['e2e']['value'])"
timeout 120 python tools/df_trace.py --batches > gpurun_out/trace_$TAG.txt 2>&1
timeout 120 python tools/kernel_times.py > gpurun_out/ktimes_$TAG.txt 2>&1
echo done
