#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "tagger or lstm or chain or full_size or sgd_step or level_paths" 2>&1 | tail -15 > gpurun_out/tests_r2g.txt
timeout 300 compute-sanitizer --tool memcheck --print-limit 10 python -c "
import sys; sys.path.insert(0,'tests'); sys.path.insert(0,'.')
import test_gpu_parity as t; t.test_tagger_small(); t.test_chain_recurrence_hidden_sizes(64, 5)" > gpurun_out/sanitizer_chain.txt 2>&1
timeout 900 python tools/config_sweep.py --only "LSTM-LM H256 V1000" --out gpurun_out/sweep_r2g.jsonl > gpurun_out/sweep_r2g.txt 2>&1
timeout 900 python tools/config_sweep.py --only "tagger" --out gpurun_out/sweep_r2g2.jsonl >> gpurun_out/sweep_r2g.txt 2>&1
echo done
