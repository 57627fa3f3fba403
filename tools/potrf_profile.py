"""Run ft_potrf (or ft_getrf / ft_geqrf) once (ABFT on or off) for an ncu
launch list; also prints host enqueue time vs device time.  Usage:
  python tools/potrf_profile.py N NB ABFT [REPS [potrf|getrf|geqrf]]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb, ft = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 1
which = sys.argv[5] if len(sys.argv) > 5 else "potrf"
A0 = si.spd_device(n, seed=7) if which == "potrf" else si.general_device(n, seed=11)
ipiv = torch.zeros(n, dtype=torch.int64, device="cuda")
tau = torch.zeros(n, dtype=torch.float64, device="cuda")
A = torch.empty_like(A0.t()).t()
ctx = abft.Context()
for r in range(reps):
    A.copy_(A0)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    a.record()
    if which == "potrf":
        rc, info, st = abft.ft_potrf(ctx, A, nb, abft=bool(ft))
    elif which == "getrf":
        rc, info, st = abft.ft_getrf(ctx, A, nb, ipiv, abft=bool(ft))
    else:
        rc, info, st = abft.ft_geqrf(ctx, A, nb, tau, abft=bool(ft))
    b.record()
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    print(f"n={n} nb={nb} abft={ft} rc={rc} info={info} dev_ms={a.elapsed_time(b):.2f} host_ms={(t1-t0)*1e3:.2f} "
          f"drv_ms={st.ms_total:.2f} checks={st.n_checks}", flush=True)
