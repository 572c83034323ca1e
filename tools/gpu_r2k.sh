#!/bin/bash
# per-warp INT_F staging (D) against the new layout with CTA-wide staging (C)
mkdir -p gpurun_out
bash tools/quick.sh warpstage
bash tools/ab.sh warpstage 3 C:C.so D:D.so
cat gpurun_out/ab_warpstage.txt
