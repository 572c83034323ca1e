#!/bin/bash
# A/B of two builds of libvpps.so on the same box (ab/A.so, ab/B.so), interleaved bench runs
TAG=${1:-ab}; N=${2:-3}
mkdir -p gpurun_out
LIB=paper_conf_micro_khorasanieas18_b200/libvpps.so
cp $LIB ab/cur.so
for i in $(seq 1 $N); do
  for v in A B; do
    cp ab/$v.so $LIB
    timeout 300 python bench.py --no-cpu-baseline --steps 200 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value']), round(d['ms_per_step']*1e3,1), round(d['roofline']['kernel_ms']*1e3,1), round(d['e2e']['value']))" >> gpurun_out/ab_$TAG.txt
  done
done
cp ab/cur.so $LIB
echo done
