#!/bin/bash
# repeat the dataflow parity tests to look for intermittent failures
mkdir -p gpurun_out
: > gpurun_out/flaky.txt
for i in 1 2 3 4 5 6; do
  timeout 300 python -m pytest tests -m gpu -q -k "dataflow or binary_target or fused_sgd" 2>&1 | grep -E "passed|failed|FAILED|Error" | head -5 >> gpurun_out/flaky.txt
done
cat gpurun_out/flaky.txt
