#!/bin/bash
# GPU tests, config-2-scale fault campaign (n=10240 nb=512, K in {1,2,4}), sweep.
mkdir -p gpurun_out
python -m pytest tests -q -m gpu -x > gpurun_out/gpu_tests.log 2>&1
tail -2 gpurun_out/gpu_tests.log
CAMPAIGN_OUT=gpurun_out/campaign_n10240.json timeout 1500 python tools/campaign.py 100 10240 512 1,2,4 potrf,getrf,geqrf > gpurun_out/campaign_n10240.log 2>&1
CAMPAIGN_OUT=gpurun_out/campaign_n10240_host.json timeout 900 python tools/campaign.py 30 10240 512 1 host_potrf,host_getrf > gpurun_out/campaign_n10240_host.log 2>&1
cat gpurun_out/campaign_n10240.log gpurun_out/campaign_n10240_host.log | grep -v Warning
timeout 1500 python tools/sweep.py > gpurun_out/sweep.log 2>&1
tail -1 gpurun_out/sweep.log
