#!/bin/bash
# Final campaigns of the round on the current tree (config 2 scale).
mkdir -p gpurun_out
CAMPAIGN_OUT=gpurun_out/campaign_n10240.json timeout 1800 python tools/campaign.py 100 10240 512 1,2,4 potrf,getrf,geqrf > gpurun_out/campaign_n10240.log 2>&1
CAMPAIGN_OUT=gpurun_out/campaign_n10240_host.json timeout 900 python tools/campaign.py 30 10240 512 1 host_potrf,host_getrf > gpurun_out/campaign_n10240_host.log 2>&1
CAMPAIGN_OUT=gpurun_out/campaign_schemes.json timeout 1800 python tools/campaign.py 100 10240 512 1 potrf,potrf:full_post,potrf:single_post,potrf:single_pre > gpurun_out/campaign_schemes.log 2>&1
cat gpurun_out/campaign_n10240.log gpurun_out/campaign_n10240_host.log gpurun_out/campaign_schemes.log | grep -v Warning
