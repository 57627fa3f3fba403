"""One encode + verify launch pair for ncu: python tools/pass_one.py N NB DTYPE(64|32) [lower]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb, bits = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
lower = len(sys.argv) > 4 and sys.argv[4] == "lower"
dt = torch.float64 if bits == 64 else torch.float32
A = si.general_device(n, seed=1, dtype=dt)
mat = abft.Mat.alloc(A, nb, mags=False)
t = abft.tiles(0, n // nb, 0, n // nb, lower, abft.SYM_LOWER if lower else abft.GENERAL)
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
for _ in range(2):
    abft.abft_encode(mat, t)
    abft.abft_verify(mat, t, abft.BOTH, tol, rep)
torch.cuda.synchronize()
print("ok", int(rep.counts.sum().item()))
