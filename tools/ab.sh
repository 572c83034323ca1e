#!/bin/bash
# A/B of builds of libvpps.so on the same box, interleaved bench runs.
#   bash tools/ab.sh TAG N [VARIANT ...]     VARIANT = name:sofile[:ENV=VAL,...]  (default A:A.so B:B.so)
TAG=${1:-ab}; N=${2:-3}; shift 2
VARS=("$@"); [ ${#VARS[@]} -eq 0 ] && VARS=(A:A.so B:B.so)
mkdir -p gpurun_out
LIB=paper_conf_micro_khorasanieas18_b200/libvpps.so
cp $LIB ab/cur.so
for i in $(seq 1 $N); do
  for v in "${VARS[@]}"; do
    IFS=: read -r name so envs <<< "$v"
    cp ab/$so $LIB
    ( [ -n "$envs" ] && export $(echo $envs | tr ',' ' '); timeout 150 python bench.py --no-cpu-baseline --steps 200 2>/dev/null ) | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$name', round(d['value']), round(d['ms_per_step']*1e3,1), round(d['roofline']['kernel_ms']*1e3,1), round(d['e2e']['value']))" >> gpurun_out/ab_$TAG.txt
  done
done
cp ab/cur.so $LIB
echo done
