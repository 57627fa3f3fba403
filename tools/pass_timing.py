"""Per-call device times of encode / verify on one matrix (CUDA events),
back to back and alternating: python tools/pass_timing.py N NB DTYPE(64|32)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb, bits = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
dt = torch.float64 if bits == 64 else torch.float32
A = si.general_device(n, seed=1, dtype=dt)
mat = abft.Mat.alloc(A, nb, mags=False)
t = abft.tiles(0, n // nb, 0, n // nb)
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
byts = n * n * (8 if bits == 64 else 4) * (1 + 4 / nb)


def one(fn):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    fn()
    b.record()
    torch.cuda.synchronize()
    return byts / (a.elapsed_time(b) / 1e3) / 1e9


enc = lambda: abft.abft_encode(mat, t)
ver = lambda: abft.abft_verify(mat, t, abft.BOTH, tol, rep)
for _ in range(3):
    enc()
    ver()
print("encode x5", [round(one(enc)) for _ in range(5)])
print("verify x5", [round(one(ver)) for _ in range(5)])
print("alternating", [(round(one(enc)), round(one(ver))) for _ in range(4)])
vc = lambda: abft.abft_verify(mat, t, abft.COL, tol, rep)
vr = lambda: abft.abft_verify(mat, t, abft.ROW, tol, rep)
ec = lambda: abft.abft_encode(mat, t, abft.COL)
er = lambda: abft.abft_encode(mat, t, abft.ROW)
print("verify COL / ROW, encode COL / ROW", [round(one(f)) for f in (vc, vr, ec, er)])
