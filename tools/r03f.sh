for e in 0 1 2; do echo "EXP $e"; VPPS_LEAF_EXP=$e timeout 60 python tools/kernel_times.py 2>&1 | grep -E "leaf_fwd|step timeline" | tail -2; done > gpurun_out/leafexp_r03f.txt 2>&1
VPPS_LEAF_EXP=1 timeout 300 ncu --set full --clock-control none -k regex:"leaf_fwd" -s 10 -c 1 -o gpurun_out/prof_r03f_e1 python bench.py --steps 2 --warmup 5 --no-cpu-baseline > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none -k regex:"leaf_fwd" -s 10 -c 1 -o gpurun_out/prof_r03f_e0 python bench.py --steps 2 --warmup 5 --no-cpu-baseline > /dev/null 2>&1
