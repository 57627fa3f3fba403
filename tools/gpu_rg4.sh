#!/bin/bash
# Device-decided restart with executable-graph updates vs the host wait (n=30720 / 20480)
mkdir -p gpurun_out; L=gpurun_out/rg4.log; : > $L
timeout 600 env ABFT_RESTART_DEVICE=1 python -m pytest tests/test_gpu_drivers.py tests/test_gpu_lu.py -q -m gpu -k "device_decided or restart" >> $L 2>&1
for mode in device host device; do
  echo "== $mode" >> $L
  if [ $mode = device ]; then export ABFT_RESTART_DEVICE=1 ABFT_DEBUG_RESTART_GRAPH=1; else unset ABFT_RESTART_DEVICE ABFT_DEBUG_RESTART_GRAPH; fi
  timeout 300 python tools/potrf_profile.py 30720 512 1 3 >> $L 2>&1
  timeout 300 python tools/lu_qr_profile.py getrf 20480 512 1 2 >> $L 2>&1
done
