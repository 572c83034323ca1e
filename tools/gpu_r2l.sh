#!/bin/bash
# vpps_df with 512 threads per CTA at H = 256 (E2, in-tree for the tests) against 256 threads (D3)
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target_config" 2>&1 | tail -3 > gpurun_out/tests_nth512.txt
cp ab/D3.so paper_conf_micro_khorasanieas18_b200/libvpps.so
timeout 400 python -m pytest tests -m gpu -q -x -k "dataflow or fused_sgd or target_config" 2>&1 | tail -3 > gpurun_out/tests_d3.txt
bash tools/ab.sh nth512b 2 D3:D3.so E2:E2.so
cat gpurun_out/tests_nth512.txt gpurun_out/tests_d3.txt gpurun_out/ab_nth512b.txt
