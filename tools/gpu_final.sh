#!/bin/bash
# Final evidence of the round on the current tree: GPU tests, smoke, bench,
# ncu launch list + full capture (reduced to CSV on the box), sweep, ft_potrf
# kernel breakdown.
mkdir -p gpurun_out/final
python __graft_entry__.py smoke > gpurun_out/final/smoke.log 2>&1; tail -1 gpurun_out/final/smoke.log
python -m pytest tests -q -m gpu > gpurun_out/final/gpu_tests.log 2>&1; tail -1 gpurun_out/final/gpu_tests.log
timeout 1200 python bench.py --steps 10 --warmup 3 > gpurun_out/final/bench.log 2>&1
tail -1 gpurun_out/final/bench.log | cut -c1-200
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final/bench_launches.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:checksum_pass -s 2 -c 2 \
   -o /tmp/prof_pass -f python bench.py --steps 1 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > /dev/null 2>&1
ncu -i /tmp/prof_pass.ncu-rep --page raw --csv > gpurun_out/final/pass_full_raw.csv 2>&1
timeout 1500 python tools/sweep.py > gpurun_out/final/sweep.log 2>&1; cp gpurun_out/sweep.json gpurun_out/final/sweep.json
python tools/potrf_profile.py 30720 512 1 3 > gpurun_out/final/potrf_times.log 2>&1
python tools/potrf_profile.py 30720 512 0 3 >> gpurun_out/final/potrf_times.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/ft.csv python tools/potrf_profile.py 30720 512 1 > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/plain.csv python tools/potrf_profile.py 30720 512 0 > /dev/null 2>&1
python tools/sum_launches.py /tmp/ft.csv > gpurun_out/final/potrf_ft_sum.txt
python tools/sum_launches.py /tmp/plain.csv > gpurun_out/final/potrf_plain_sum.txt
ls gpurun_out/final
