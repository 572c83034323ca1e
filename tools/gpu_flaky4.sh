#!/bin/bash
# localise the intermittent corruption: 20 repeats per variant, count runs with any ratio > 1e-4
mkdir -p gpurun_out
: > gpurun_out/flaky4.txt
run() { # name so env
  cp ab/$2.so paper_conf_micro_khorasanieas18_b200/libvpps.so
  ( [ -n "$3" ] && export $3; timeout 600 python tools/flaky_diag.py 5 20 > gpurun_out/fl_$1.txt 2>&1 )
  echo "$1 bad=$(grep -c 'e-0[1-4] ' gpurun_out/fl_$1.txt) runs=$(grep -c '^run' gpurun_out/fl_$1.txt)" >> gpurun_out/flaky4.txt
}
run F F ""
run F_coop F VPPS_DF_COOP=1
run F_nopdl F VPPS_DF_NOPDL=1
run C C ""
run C_nopdl C VPPS_DF_NOPDL=1
run A A ""
cp ab/F.so paper_conf_micro_khorasanieas18_b200/libvpps.so
cat gpurun_out/flaky4.txt
