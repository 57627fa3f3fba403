"""Per-iteration main-stream time of a driver, unprotected vs ABFT (one run
each after a warm-up; the library prints the per-iteration ms to stderr when
ABFT_ITER_EVENTS=1).  Usage:
  ABFT_ITER_EVENTS=1 python tools/iter_time.py [N NB [potrf|getrf|geqrf]]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n = int(sys.argv[1]) if len(sys.argv) > 1 else 30720
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 512
which = sys.argv[3] if len(sys.argv) > 3 else "potrf"
A0 = si.spd_device(n, seed=7) if which == "potrf" else si.general_device(n, seed=11)
ipiv = torch.zeros(n, dtype=torch.int64, device="cuda")
tau = torch.zeros(n, dtype=torch.float64, device="cuda")
A = torch.empty_like(A0.t()).t()
ctx = abft.Context()
for tag, ft in (("warm", True), ("plain", False), ("ft", True)):
    A.copy_(A0)
    torch.cuda.synchronize()
    print(f"== {tag}", file=sys.stderr, flush=True)
    if which == "potrf":
        rc, info, st = abft.ft_potrf(ctx, A, nb, abft=ft)
    elif which == "getrf":
        rc, info, st = abft.ft_getrf(ctx, A, nb, ipiv, abft=ft)
    else:
        rc, info, st = abft.ft_geqrf(ctx, A, nb, tau, abft=ft)
    torch.cuda.synchronize()
    assert rc == 0 and info == 0
