#!/bin/bash
mkdir -p gpurun_out
python tools/gemm_bench.py > gpurun_out/gemm_r2f.txt 2>&1
VPPS_GEMM_TC_MIN=-1 python tools/gemm_bench.py >> gpurun_out/gemm_r2f.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"vpps_dw_tc" -s 4 -c 1 -o gpurun_out/prof_dwtc python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_dwtc.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"tc_sgemm" -s 3 -c 1 -o gpurun_out/prof_tcg python tools/gemm_bench.py > /dev/null 2>&1
echo done
