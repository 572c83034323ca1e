mkdir -p gpurun_out
bash tools/quick.sh r03c
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"leaf_fwd|dw_gemm" -s 10 -c 2 -o gpurun_out/prof_r03c python bench.py --steps 2 --warmup 5 --no-cpu-baseline > gpurun_out/ncu_r03c.log 2>&1
