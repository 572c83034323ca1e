#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/tests_r2g.txt
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2g.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_r2g.txt
timeout 300 python bench.py > gpurun_out/bench_r2g.json 2> gpurun_out/bench_r2g.err
cat gpurun_out/tests_r2g.txt gpurun_out/smoke_r2g.txt; python -c "import json; d=json.load(open('gpurun_out/bench_r2g.json')); print(d['value'], d['ms_per_step'], d['roofline']['kernel_ms'], d['e2e']['value'])"
