#!/bin/bash
mkdir -p gpurun_out
python -m pytest tests -q -m gpu > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
timeout 600 python tools/multi_fault_repro.py geqrf 2048 256 2 150 > gpurun_out/mfr_qr_2048.log 2>&1; tail -1 gpurun_out/mfr_qr_2048.log
CAMPAIGN_OUT=gpurun_out/campaign_n10240.json timeout 1800 python tools/campaign.py 100 10240 512 1,2,4 potrf,getrf,geqrf > gpurun_out/campaign_n10240.log 2>&1
CAMPAIGN_OUT=gpurun_out/campaign_n10240_host.json timeout 900 python tools/campaign.py 30 10240 512 1 host_potrf,host_getrf > gpurun_out/campaign_n10240_host.log 2>&1
cat gpurun_out/campaign_n10240.log gpurun_out/campaign_n10240_host.log | grep -v Warning
