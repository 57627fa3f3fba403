#!/bin/bash
set -x
mkdir -p gpurun_out
python -m pytest tests -q -m gpu > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
python tools/potrf_profile.py 30720 512 1 3 > gpurun_out/potrf_times.log 2>&1
python tools/potrf_profile.py 30720 512 0 3 >> gpurun_out/potrf_times.log 2>&1
cat gpurun_out/potrf_times.log | grep n=
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/potrf_ft_launches.csv python tools/potrf_profile.py 10240 512 1 > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/potrf_plain_launches.csv python tools/potrf_profile.py 10240 512 0 > /dev/null 2>&1
python tools/sum_launches.py gpurun_out/potrf_ft_launches.csv > gpurun_out/potrf_ft_sum.txt
python tools/sum_launches.py gpurun_out/potrf_plain_launches.csv > gpurun_out/potrf_plain_sum.txt
head -25 gpurun_out/potrf_ft_sum.txt
