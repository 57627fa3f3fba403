#!/bin/bash
# Full GPU session: smoke, all GPU tests, bench (N=1), launch list.
set -x
mkdir -p gpurun_out
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
tail -2 gpurun_out/smoke.log
python -m pytest tests -q -m gpu > gpurun_out/gpu_tests.log 2>&1
tail -4 gpurun_out/gpu_tests.log
timeout 1200 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.log 2>&1
tail -1 gpurun_out/bench.log
