"""Quick driver timing (CUDA events, median of reps): ft_* with ABFT (with and
without local restart) vs the same driver unprotected, plus the cuSOLVER
factorization as context.  Usage:
  python tools/drv_time.py potrf|getrf|geqrf N NB [REPS] [host]
("host": the panel decomposition on the host LAPACK, FT_PD_HOST)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

which, n, nb = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
host = len(sys.argv) > 5 and sys.argv[5] == "host"
A0 = si.spd_device(n, seed=7) if which == "potrf" else si.general_device(n, seed=11)
A = torch.empty_like(A0.t()).t()
ctx = abft.Context()
kw = {}
if host:
    ctx.set_host_lapack()
    kw = {"pd_location": abft.PD_HOST}
ipiv = torch.zeros(n, dtype=torch.int64, device="cuda")
tau = torch.zeros(n, dtype=torch.float64, device="cuda")


def run(ft, restart=True, la=True):
    A.copy_(A0)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    if which == "potrf":
        rc, info, st = abft.ft_potrf(ctx, A, nb, abft=ft, restart=restart, lookahead=la, **kw)
    elif which == "getrf":
        rc, info, st = abft.ft_getrf(ctx, A, nb, ipiv, abft=ft, restart=restart, **kw)
    else:
        rc, info, st = abft.ft_geqrf(ctx, A, nb, tau, abft=ft, restart=restart, **kw)
    b.record()
    torch.cuda.synchronize()
    assert rc == 0 and info == 0 and sum(st.counts) == 0, (rc, info, list(st.counts))
    return a.elapsed_time(b)


def med(f):
    f()
    ts = sorted(f() for _ in range(reps))
    return ts[len(ts) // 2]


plain = med(lambda: run(False))
ft = med(lambda: run(True))
nors = med(lambda: run(True, restart=False))
if which == "potrf":
    p0, f0 = med(lambda: run(False, la=False)), med(lambda: run(True, la=False))
    print(f"potrf without look-ahead: plain {p0:.2f} ms, ft {f0:.2f} ms ({100 * (f0 - p0) / p0:.2f}%)")
S = A0.t().contiguous()
torch.backends.cuda.preferred_linalg_library("cusolver")
lib = {"potrf": lambda: torch.linalg.cholesky(S), "getrf": lambda: torch.linalg.lu_factor(S),
       "geqrf": lambda: torch.geqrf(S)}[which]


def tl():
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    lib()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b)


cus = med(tl)
print(f"{which}{' host-PD' if host else ''} n={n} nb={nb}: plain {plain:.2f} ms, ft {ft:.2f} ms ({100 * (ft - plain) / plain:.2f}%), "
      f"ft no-restart {nors:.2f} ms ({100 * (nors - plain) / plain:.2f}%), cusolver {cus:.2f} ms "
      f"(ft vs cusolver {100 * (ft - cus) / cus:.2f}%)", flush=True)
if which == "potrf" and not host:
    A.copy_(A0)
    rc, info, st = abft.ft_potrf(ctx, A, nb, timing=True)
    torch.cuda.synchronize()
    print("phase ms (timing run; side-stream phases overlap the main stream):",
          {k: round(v, 2) for k, v in zip(abft.PHASES, st.ms_phase)})
