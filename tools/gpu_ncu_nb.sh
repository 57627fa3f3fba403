#!/bin/bash
set -x
mkdir -p gpurun_out
for cfg in "32768 256 64" "32768 1024 64" "32768 512 64" "32768 256 32"; do
  set -- $cfg
  timeout 600 ncu --set full --clock-control none -k regex:checksum_pass -s 2 -c 2 -o gpurun_out/prof_${1}_${2}_${3} -f python tools/pass_one.py $1 $2 $3 > gpurun_out/ncu_${1}_${2}_${3}.log 2>&1
done
ls gpurun_out/
