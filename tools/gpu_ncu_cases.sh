#!/bin/bash
# ncu --set full captures of single encode/verify launches for the sweep's weak
# configurations (python tools/pass_one.py N NB BITS [lower]); the reports are
# reduced to raw-page CSVs on the box (gpurun copies back <= 64 MiB).
mkdir -p gpurun_out/ncu_cases
for cfg in "$@"; do
  set -- $cfg
  tag=$(echo "$cfg" | tr ' ' '_')
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:checksum_pass -s 2 -c 2 \
    -o /tmp/prof_$tag -f python tools/pass_one.py $cfg > gpurun_out/ncu_cases/$tag.log 2>&1
  ncu -i /tmp/prof_$tag.ncu-rep --page raw --csv > gpurun_out/ncu_cases/$tag.raw.csv 2>&1
  ncu -i /tmp/prof_$tag.ncu-rep --page details --csv > gpurun_out/ncu_cases/$tag.details.csv 2>&1
  tail -1 gpurun_out/ncu_cases/$tag.log
done
