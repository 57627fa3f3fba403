"""Run ft_getrf / ft_geqrf once (ABFT on or off) for an ncu launch list.
Usage: python tools/lu_qr_profile.py {getrf|geqrf} N NB ABFT [reps]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

which, n, nb, ft = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 1
A0 = si.general_device(n, seed=21)
A = torch.empty_like(A0.t()).t()
ctx = abft.Context()
ipiv = torch.zeros(n, dtype=torch.int64, device="cuda")
tau = torch.zeros(n, dtype=torch.float64, device="cuda")
for r in range(reps):
    A.copy_(A0)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    if which == "getrf":
        rc, info, st = abft.ft_getrf(ctx, A, nb, ipiv, abft=bool(ft))
    else:
        rc, info, st = abft.ft_geqrf(ctx, A, nb, tau, abft=bool(ft))
    b.record()
    torch.cuda.synchronize()
    print(f"{which} n={n} nb={nb} abft={ft} rc={rc} dev_ms={a.elapsed_time(b):.2f} checks={st.n_checks} "
          f"counts={list(st.counts)}", flush=True)
