#!/bin/bash
# round 2, session 4: unit-pair x column-slice register layout of vpps_df (B: one node per transposed step,
# C: two) against the previous layout (A)
mkdir -p gpurun_out
bash tools/quick.sh flip
bash tools/ab.sh flip 3 A:A.so B:B.so C:C.so
cat gpurun_out/ab_flip.txt
