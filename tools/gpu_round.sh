#!/bin/bash
# Round evidence (run under gpurun from the repo root): smoke, every GPU
# test, the N=1 bench line, the ncu launch list of the bench step and of one
# ft_potrf, one ncu --set full capture of the checksum pass (compute-sanitizer
# is closed on the GPU pool).
#   gpurun --timeout 3600 -- 'bash tools/gpu_round.sh r02'
tag=${1:-round}
out=gpurun_out/$tag
mkdir -p $out
python __graft_entry__.py smoke > $out/smoke.log 2>&1; tail -1 $out/smoke.log
timeout 2400 python -m pytest tests -q -m gpu > $out/gpu_tests.log 2>&1; tail -1 $out/gpu_tests.log
timeout 1500 python bench.py --steps 10 --warmup 3 > $out/bench.log 2>&1
tail -1 $out/bench.log | cut -c1-300
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/bench_launches.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu > $out/ncu_launch.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none -c 6000 --csv \
   --log-file $out/potrf30720_launches.csv python tools/potrf_profile.py 30720 512 1 > $out/potrf_prof.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none -c 6000 --csv \
   --log-file $out/potrf30720_plain_launches.csv python tools/potrf_profile.py 30720 512 0 > $out/potrf_prof0.log 2>&1
for ft in 0 1; do
  timeout 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none -c 8000 --csv \
     --log-file $out/getrf20480_ft${ft}_launches.csv python tools/potrf_profile.py 20480 512 $ft 1 getrf > /dev/null 2>&1
done
python tools/drv_time.py potrf 30720 512 3 > $out/drv_potrf.log 2>&1
python tools/drv_time.py getrf 20480 512 3 > $out/drv_getrf.log 2>&1
python tools/drv_time.py geqrf 20480 512 3 > $out/drv_geqrf.log 2>&1
python tools/drv_time.py getrf 20480 512 3 host > $out/drv_getrf_host.log 2>&1
python tools/rule_time.py > $out/rule_time.log 2>&1
ABFT_RULE_CUBLAS=1 python tools/rule_time.py >> $out/rule_time.log 2>&1
ABFT_ITER_EVENTS=1 python tools/iter_time.py 30720 512 potrf 2> $out/iter_potrf.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:checksum_pass -s 2 -c 2 \
   -o $out/prof_pass -f python bench.py --steps 1 --warmup 1 --no-e2e --no-potrf --no-cpu --no-lu-qr --no-mgpu \
   > $out/ncu_full.log 2>&1
for sk in 0 1 2 3 7 15; do ABFT_DIAG_SKIP=$sk python tools/diag_time.py 30720 512 3 2>&1 | grep skip; done > $out/diag_skip.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dmma -s 1 -c 1 -o $out/prof_rule -f \
   python tools/rule_ncu.py 59 > $out/ncu_rule.log 2>&1
python tools/small_pass.py > $out/small_pass.log 2>&1
