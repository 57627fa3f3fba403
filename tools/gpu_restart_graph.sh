#!/bin/bash
# Device-decided local restart (graph IF node) vs the host round trip:
# ft_potrf n=30720 and ft_getrf n=20480 timings with both.
mkdir -p gpurun_out
L=gpurun_out/restart_graph.log
: > $L
for mode in graph host graph; do
  if [ $mode = host ]; then export ABFT_RESTART_HOST_WAIT=1; else unset ABFT_RESTART_HOST_WAIT; fi
  echo "== $mode" >> $L
  timeout 300 python tools/potrf_profile.py 30720 512 1 4 >> $L 2>&1
  timeout 300 python tools/lu_qr_profile.py getrf 20480 512 1 3 >> $L 2>&1
done
unset ABFT_RESTART_HOST_WAIT
echo "== plain" >> $L
timeout 300 python tools/potrf_profile.py 30720 512 0 3 >> $L 2>&1
timeout 300 python tools/lu_qr_profile.py getrf 20480 512 0 3 >> $L 2>&1
