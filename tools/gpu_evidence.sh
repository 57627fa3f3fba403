#!/bin/bash
# Round evidence: smoke, all GPU tests, the N=1 bench line, the ncu launch list
# of the bench's checksum pass, one ncu --set full capture of the dominant kernel.
set -x
mkdir -p gpurun_out
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
tail -1 gpurun_out/smoke.log
python -m pytest tests -q -m gpu > gpurun_out/gpu_tests.log 2>&1
tail -2 gpurun_out/gpu_tests.log
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu_info.txt
timeout 1500 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.log 2>&1
tail -1 gpurun_out/bench.log | cut -c1-400
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:checksum_pass -s 2 -c 2 \
   -o gpurun_out/prof_pass -f python bench.py --steps 1 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log
