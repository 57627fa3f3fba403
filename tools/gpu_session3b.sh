#!/bin/bash
mkdir -p gpurun_out
for s in 0 1 2 4 8; do ABFT_NSLAB=$s timeout 300 python tools/slab_tune.py > gpurun_out/slab_tune_$s.log 2>&1; done
grep -h "tiles=" gpurun_out/slab_tune_*.log | sort -t= -k3 -n | head -80
CAMPAIGN_OUT=gpurun_out/campaign_n10240.json timeout 1800 python tools/campaign.py 100 10240 512 1,2,4 potrf,getrf,geqrf > gpurun_out/campaign_n10240.log 2>&1
CAMPAIGN_OUT=gpurun_out/campaign_n10240_host.json timeout 900 python tools/campaign.py 30 10240 512 1 host_potrf,host_getrf > gpurun_out/campaign_n10240_host.log 2>&1
cat gpurun_out/campaign_n10240.log gpurun_out/campaign_n10240_host.log | grep -v Warning
