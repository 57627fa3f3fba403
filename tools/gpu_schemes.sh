#!/bin/bash
# checking-scheme parity tests, scheme campaign (Table VIII analogue), bench (overheads per scheme)
mkdir -p gpurun_out
python -m pytest tests/test_gpu_schemes.py tests/test_gpu_drivers.py -q > gpurun_out/t_schemes.log 2>&1; tail -3 gpurun_out/t_schemes.log
CAMPAIGN_OUT=gpurun_out/campaign_schemes.json timeout 1800 python tools/campaign.py 100 10240 512 1 potrf,potrf:full_post,potrf:single_post,potrf:single_pre > gpurun_out/campaign_schemes.log 2>&1
grep -v Warning gpurun_out/campaign_schemes.log
timeout 1200 python bench.py --steps 10 --warmup 3 --no-lu-qr --no-mgpu --no-cpu --no-e2e > gpurun_out/bench_schemes.log 2>&1
tail -1 gpurun_out/bench_schemes.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ft_potrf'])"
