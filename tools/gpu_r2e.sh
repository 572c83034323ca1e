#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target or dp_ or sgd_step or tensor_core" 2>&1 | tail -15 > gpurun_out/tests_r2e.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" >> gpurun_out/tests_r2e.txt 2>&1
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_r2e.json 2> gpurun_out/bench_r2e.err
timeout 120 python tools/kernel_times.py > gpurun_out/ktimes_r2e.txt 2>&1
echo done
