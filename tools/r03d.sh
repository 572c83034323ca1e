for e in 0 1 2 3; do echo "EXP $e"; VPPS_LEAF_EXP=$e timeout 120 python tools/kernel_times.py 2>&1 | grep -E "leaf_fwd|step timeline" | tail -3; done > gpurun_out/leafexp_r03d.txt 2>&1
for e in 0 1 2 3; do echo "EXP $e NOFLUSH"; VPPS_LEAF_EXP=$e timeout 120 python tools/kernel_times.py --no-flush 2>&1 | grep -E "leaf_fwd" | tail -1; done >> gpurun_out/leafexp_r03d.txt 2>&1
