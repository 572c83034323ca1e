#!/bin/bash
# bounds-checked vpps_df (VPPS_DF_CHECK=1: every batch entry against its region, trap on violation) on every
# dataflow GPU test and a bench run — the pool's replacement for a compute-sanitizer pass
#   build: VPPS_NVCC_EXTRA="-DVPPS_DF_CHECK=1" python -c "import __graft_entry__ as g; g.build()"; cp ... ab/CHK.so
TAG=${1:-chk}
mkdir -p gpurun_out
cp paper_conf_micro_khorasanieas18_b200/libvpps.so ab/prod.so
cp ab/CHK.so paper_conf_micro_khorasanieas18_b200/libvpps.so
timeout 900 python -m pytest tests -m gpu -q -k "dataflow or target or binary or fused_sgd or sgd_step or dp_two" 2>&1 | tail -4 > gpurun_out/checked_$TAG.txt
timeout 300 python bench.py --no-cpu-baseline --steps 50 >> gpurun_out/checked_$TAG.txt 2>&1; echo "bench rc=$?" >> gpurun_out/checked_$TAG.txt
cp ab/prod.so paper_conf_micro_khorasanieas18_b200/libvpps.so
cat gpurun_out/checked_$TAG.txt
