#!/bin/bash
set -x
mkdir -p gpurun_out
python -m pytest tests/test_gpu_checksum.py tests/test_gpu_drivers.py -q -x > gpurun_out/gpu_tests_ck.log 2>&1
tail -3 gpurun_out/gpu_tests_ck.log
SWEEP_N=16384,32768,65536 timeout 1200 python tools/sweep.py > gpurun_out/sweep.log 2>&1
python - <<'PY'
import json
rows=json.load(open('gpurun_out/sweep.json'))
for r in rows:
    print(f"{r['dtype']:8s} {r['n']:6d} {r['nb']:5d} {str(r['lower_only'])[0]:>4s} {r['encode_GBs']:7.0f} {r['verify_GBs']:7.0f} {r['encode_verify_GBs']:7.0f} {r.get('gemm_prior_art_GBs',0):7.0f}")
PY
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-lu-qr --potrf-reps 1 > gpurun_out/bench_q.log 2>&1
tail -1 gpurun_out/bench_q.log | cut -c1-200
