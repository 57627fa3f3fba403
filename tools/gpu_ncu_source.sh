#!/bin/bash
# ncu full capture of one pass_one.py configuration, reduced on the box to the
# source page (per-line samples) and the raw page.
mkdir -p gpurun_out/ncu_src
tag=$(echo "$*" | tr ' ' '_')
timeout 600 ncu --set full --clock-control none --import-source on -k regex:checksum_pass -s ${NCU_SKIP:-2} -c 1 \
  -o /tmp/prof_src -f python tools/pass_one.py "$@" > gpurun_out/ncu_src/$tag.log 2>&1
ncu -i /tmp/prof_src.ncu-rep --page source --csv > gpurun_out/ncu_src/$tag.source.csv 2>&1
ncu -i /tmp/prof_src.ncu-rep --page raw --csv > gpurun_out/ncu_src/$tag.raw.csv 2>&1
ls -la gpurun_out/ncu_src
