"""Marginal cost of each class of ABFT work in ft_potrf (timing diagnostics):
run under ABFT_DIAG_SKIP=<bits> (ft_driver.cuh: 1 main-stream checks, 2
side-stream checks, 4 TMU rule, 8 PD/PU rules) and compare the medians.
  ABFT_DIAG_SKIP=3 python tools/diag_time.py N NB [REPS]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb = int(sys.argv[1]), int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
A0 = si.spd_device(n, seed=7)
A = torch.empty_like(A0.t()).t()
ctx = abft.Context()


def run(ft, restart):
    A.copy_(A0)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    rc, info, st = abft.ft_potrf(ctx, A, nb, abft=ft, restart=restart)
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b)


def med(ft, restart):
    run(ft, restart)
    ts = sorted(run(ft, restart) for _ in range(reps))
    return ts[len(ts) // 2]


plain = med(False, False)
ft = med(True, True)
ftnr = med(True, False)
print(f"skip={os.environ.get('ABFT_DIAG_SKIP', '0')} plain {plain:.2f} ft {ft:.2f} (+{ft - plain:.2f} ms) "
      f"ft-no-restart {ftnr:.2f} (+{ftnr - plain:.2f} ms)", flush=True)
