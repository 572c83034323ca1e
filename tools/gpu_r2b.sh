#!/bin/bash
# round-2 check: full -m gpu suite, smoke, sanitizers on one small pass per path
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/tests_r2b.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2b.txt 2>&1
for tool in memcheck racecheck synccheck; do
  for path in dataflow level grid; do
    echo "== $tool $path" >> gpurun_out/sanitizer_r2b.txt
    timeout 600 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_pass.py $path >> gpurun_out/sanitizer_r2b.txt 2>&1
    echo "rc=$?" >> gpurun_out/sanitizer_r2b.txt
  done
done
echo done
