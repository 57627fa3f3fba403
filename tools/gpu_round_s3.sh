#!/bin/bash
# Round evidence (session 3): smoke, bench N=1, ncu launch list + full capture
# of the checksum pass (reduced to CSV on the box), ft_potrf kernel breakdown.
mkdir -p gpurun_out/s3
python __graft_entry__.py smoke > gpurun_out/s3/smoke.log 2>&1; tail -1 gpurun_out/s3/smoke.log
python -m pytest tests -q -m gpu > gpurun_out/s3/gpu_tests.log 2>&1; tail -1 gpurun_out/s3/gpu_tests.log
timeout 1200 python bench.py --steps 10 --warmup 3 > gpurun_out/s3/bench.log 2>&1
tail -1 gpurun_out/s3/bench.log | cut -c1-300
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s3/bench_launches.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > gpurun_out/s3/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:checksum_pass -s 2 -c 2 \
   -o /tmp/prof_pass -f python bench.py --steps 1 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > gpurun_out/s3/ncu_full.log 2>&1
ncu -i /tmp/prof_pass.ncu-rep --page raw --csv > gpurun_out/s3/pass_full_raw.csv 2>&1
ncu -i /tmp/prof_pass.ncu-rep --page details --csv > gpurun_out/s3/pass_full_details.csv 2>&1
python tools/potrf_profile.py 30720 512 1 3 > gpurun_out/s3/potrf_times.log 2>&1
python tools/potrf_profile.py 30720 512 0 3 >> gpurun_out/s3/potrf_times.log 2>&1
grep n= gpurun_out/s3/potrf_times.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s3/potrf_ft_launches.csv python tools/potrf_profile.py 30720 512 1 > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s3/potrf_plain_launches.csv python tools/potrf_profile.py 30720 512 0 > /dev/null 2>&1
python tools/sum_launches.py gpurun_out/s3/potrf_ft_launches.csv > gpurun_out/s3/potrf_ft_sum.txt
python tools/sum_launches.py gpurun_out/s3/potrf_plain_launches.csv > gpurun_out/s3/potrf_plain_sum.txt
rm -f gpurun_out/s3/potrf_ft_launches.csv gpurun_out/s3/potrf_plain_launches.csv
head -30 gpurun_out/s3/potrf_ft_sum.txt
