#!/bin/bash
set -x
mkdir -p gpurun_out
python -m pytest tests/test_gpu_lu.py tests/test_gpu_qr.py -q -x > gpurun_out/gpu_tests_qrlu.log 2>&1
tail -3 gpurun_out/gpu_tests_qrlu.log
timeout 900 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --potrf-reps 1 --lu-qr-reps 2 > gpurun_out/bench_luqr.log 2>&1
tail -1 gpurun_out/bench_luqr.log
timeout 1200 python tools/sweep.py > gpurun_out/sweep.log 2>&1
tail -3 gpurun_out/sweep.log
