"""Per-phase host time of the FT_PD_HOST drivers (ABFT_HOST_TIMING=1 prints
the split to stderr): potrf n=30720, getrf/geqrf n=20480, ABFT on and off."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["ABFT_HOST_TIMING"] = "1"
import synth_inputs as si  # noqa: E402
from paper_conf_sc_chenlllwtolzgc18_b200 import abft  # noqa: E402

ctx = abft.Context()
ctx.set_host_lapack()
nb = 512


def timed(fn):
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    rc, info, st = fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b), st


A0 = si.spd_device(30720, seed=7)
A = torch.empty_like(A0.t()).t()
for ft in (True, False, True, False):
    A.copy_(A0)
    ms, st = timed(lambda: abft.ft_potrf(ctx, A, nb, abft=ft, pd_location=abft.PD_HOST))
    print(f"potrf ft={ft} {ms:.1f} ms host {st.ms_host_pd:.1f}", flush=True)
del A, A0
G0 = si.general_device(20480, seed=21)
G = torch.empty_like(G0.t()).t()
ipiv = torch.zeros(20480, dtype=torch.int64, device="cuda")
tau = torch.zeros(20480, dtype=torch.float64, device="cuda")
for name, f in [("getrf", lambda ft: abft.ft_getrf(ctx, G, nb, ipiv, abft=ft, pd_location=abft.PD_HOST)),
                ("geqrf", lambda ft: abft.ft_geqrf(ctx, G, nb, tau, abft=ft, pd_location=abft.PD_HOST))]:
    for ft in (True, False):
        G.copy_(G0)
        ms, st = timed(lambda: f(ft))
        print(f"{name} ft={ft} {ms:.1f} ms host {st.ms_host_pd:.1f}", flush=True)
