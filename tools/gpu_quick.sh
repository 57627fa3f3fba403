#!/bin/bash
set -x
mkdir -p gpurun_out
python -m pytest tests -q -m gpu -x > gpurun_out/gpu_tests.log 2>&1
tail -2 gpurun_out/gpu_tests.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-lu-qr --potrf-reps 3 > gpurun_out/bench_q.log 2>&1
tail -1 gpurun_out/bench_q.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline'], d['ft_potrf'], d['clocks'])"
[ -n "$SWEEP" ] && SWEEP_N=32768 timeout 1200 python tools/sweep.py > gpurun_out/sweep.log 2>&1
[ -n "$SWEEP" ] && python - <<'PY'
import json
rows=json.load(open('gpurun_out/sweep.json'))
for r in rows:
    print(f"{r['dtype']:8s} {r['n']:6d} {r['nb']:5d} {str(r['lower_only'])[0]:>4s} {r['encode_GBs']:7.0f} {r['verify_GBs']:7.0f} {r['encode_verify_GBs']:7.0f} {r.get('gemm_prior_art_GBs',0):7.0f}")
PY
