"""Run ft_potrf once (ABFT on or off) for an ncu launch list; also prints host
enqueue time vs device time.  Usage: python tools/potrf_profile.py N NB ABFT"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb, ft = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 1
A0 = si.spd_device(n, seed=7)
A = torch.empty_like(A0.t()).t()
ctx = abft.Context()
for r in range(reps):
    A.copy_(A0)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    a.record()
    rc, info, st = abft.ft_potrf(ctx, A, nb, abft=bool(ft))
    b.record()
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    print(f"n={n} nb={nb} abft={ft} rc={rc} info={info} dev_ms={a.elapsed_time(b):.2f} host_ms={(t1-t0)*1e3:.2f} "
          f"drv_ms={st.ms_total:.2f} checks={st.n_checks}", flush=True)
