#!/bin/bash
set -x
mkdir -p gpurun_out
python -m pytest tests/test_gpu_checksum.py -q -x > gpurun_out/gpu_tests_ck.log 2>&1
tail -3 gpurun_out/gpu_tests_ck.log
timeout 1200 python tools/sweep.py > gpurun_out/sweep.log 2>&1
python - <<'PY'
import json
rows=json.load(open('gpurun_out/sweep.json'))
for r in rows:
    print(f"{r['dtype']:8s} {r['n']:6d} {r['nb']:5d} {str(r['lower_only'])[0]:>4s} {r['encode_GBs']:7.0f} {r['verify_GBs']:7.0f} {r['encode_verify_GBs']:7.0f} {r.get('gemm_prior_art_GBs',0):7.0f}")
PY
