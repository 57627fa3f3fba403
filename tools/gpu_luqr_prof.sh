#!/bin/bash
set -x
mkdir -p gpurun_out
for w in getrf geqrf; do
  for f in 1 0; do
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${w}_${f}_launches.csv python tools/lu_qr_profile.py $w 20480 512 $f > /dev/null 2>&1
    python tools/sum_launches.py gpurun_out/${w}_${f}_launches.csv > gpurun_out/${w}_${f}_sum.txt
  done
done
head -20 gpurun_out/getrf_1_sum.txt; tail -1 gpurun_out/getrf_0_sum.txt
head -20 gpurun_out/geqrf_1_sum.txt; tail -1 gpurun_out/geqrf_0_sum.txt
