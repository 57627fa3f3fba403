"""One Cholesky TMU-rule launch (fp64 DMMA kernel) at ntk (default 59) for
an ncu --set full capture:  python tools/rule_ncu.py [NTK]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_sc_chenlllwtolzgc18_b200 import abft

nb, ntk = 512, int(sys.argv[1]) if len(sys.argv) > 1 else 59
nk = ntk * nb
L = torch.randn(nb, nk, device="cuda", dtype=torch.float64).t()
cL = torch.randn(nb, 2 * ntk, device="cuda", dtype=torch.float64).t()
mL = torch.rand(nb, ntk, device="cuda", dtype=torch.float64).t()
Cc = torch.zeros(nk, 2 * ntk, device="cuda", dtype=torch.float64).t()
Rr = torch.zeros(2 * ntk, nk, device="cuda", dtype=torch.float64).t()
Cm = torch.zeros(nk, ntk, device="cuda", dtype=torch.float64).t()
Rm = torch.zeros(ntk, nk, device="cuda", dtype=torch.float64).t()
for _ in range(2):
    abft.abft_update_syrk(nb, ntk, L, cL, Cc, Rr, mL, Cm, Rm)
torch.cuda.synchronize()
