#!/bin/bash
set -x
mkdir -p gpurun_out
python -m pytest tests/test_gpu_qr.py tests/test_gpu_lu.py -q -x > gpurun_out/gpu_tests_qrlu.log 2>&1
tail -15 gpurun_out/gpu_tests_qrlu.log
