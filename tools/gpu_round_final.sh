#!/bin/bash
# Full evidence session: smoke, all GPU tests, bench (N=1), ncu launch list + full capture, sweep, campaign.
set -x
mkdir -p gpurun_out
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
tail -1 gpurun_out/smoke.log
python -m pytest tests -q -m gpu > gpurun_out/gpu_tests.log 2>&1
tail -2 gpurun_out/gpu_tests.log
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu_info.txt
timeout 1200 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.log 2>&1
tail -1 gpurun_out/bench.log | cut -c1-300
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:checksum_pass -s 2 -c 2 \
   -o gpurun_out/prof_pass -f python bench.py --steps 1 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > gpurun_out/ncu_full.log 2>&1
timeout 1500 python tools/sweep.py > gpurun_out/sweep.log 2>&1
timeout 1200 python tools/campaign.py 40 1024 128 > gpurun_out/campaign.log 2>&1
tail -4 gpurun_out/campaign.log
