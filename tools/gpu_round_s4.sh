#!/bin/bash
# Round evidence (session 4): smoke, full GPU suite, bench N=1, ncu launch list
# of the bench step.
mkdir -p gpurun_out/s4
python __graft_entry__.py smoke > gpurun_out/s4/smoke.log 2>&1; tail -1 gpurun_out/s4/smoke.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/s4/gpu_tests.log 2>&1; tail -1 gpurun_out/s4/gpu_tests.log
timeout 1200 python bench.py --steps 10 --warmup 3 > gpurun_out/s4/bench.log 2>&1
tail -1 gpurun_out/s4/bench.log | cut -c1-400
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s4/bench_launches.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > gpurun_out/s4/ncu_launch.log 2>&1
