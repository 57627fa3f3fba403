"""Single small checksum pass for an ncu capture: python tools/pass_small_ncu.py NTILES"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

ntiles = int(sys.argv[1])
n, nb = 30720, 512
nt = n // nb
A = si.spd_device(n, seed=3)
mat = abft.Mat.alloc(A, nb)
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
abft.abft_encode(mat, abft.tiles(0, nt, 0, nt))
tl = abft.tiles(nt - ntiles, nt, 0, 1)
for _ in range(3):
    abft.abft_verify(mat, tl, abft.COL, tol, rep)
torch.cuda.synchronize()
