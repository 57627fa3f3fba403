"""The driver's small per-iteration launches in isolation, for an ncu capture
(`ncu --set full -k regex:"checksum_pass|locate|dmma"`): each op is called
twice, cold and warm.  n=30720 nb=512 fp64 shapes of ft_potrf.
  python tools/small_probe.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb = 30720, 512
nt = n // nb
A = si.spd_device(n, seed=3)
mat = abft.Mat.alloc(A, nb)
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
abft.abft_encode(mat, abft.tiles(0, nt, 0, nt, True, abft.SYM_LOWER))
fixes = torch.zeros(64 * abft.FIX_BYTES, dtype=torch.uint8, device="cuda")
nfx = torch.zeros(1, dtype=torch.int32, device="cuda")
torch.cuda.synchronize()
k = 30
ops = [
    ("verify 1 tile SYM both", lambda: abft.abft_verify(mat, abft.tiles(k, k + 1, k, k + 1, False, abft.SYM_LOWER),
                                                         abft.BOTH, tol, rep)),
    ("verify 1 tile LOWER col", lambda: abft.abft_verify(mat, abft.tiles(k, k + 1, k, k + 1, False, abft.LOWER),
                                                          abft.COL, tol, rep)),
    ("verify panel both", lambda: abft.abft_verify(mat, abft.tiles(k + 1, nt, k, k + 1), abft.BOTH, tol, rep)),
    ("verify panel col", lambda: abft.abft_verify(mat, abft.tiles(k + 1, nt, k, k + 1), abft.COL, tol, rep)),
    ("locate panel", lambda: abft.abft_locate_correct(mat, abft.tiles(k + 1, nt, k, k + 1), abft.COL, tol, rep,
                                                       fixes, nfx)),
]
ntk = 5
L = torch.randn(nb, ntk * nb, device="cuda", dtype=torch.float64).t()
cL = torch.randn(nb, 2 * ntk, device="cuda", dtype=torch.float64).t()
mL = torch.rand(nb, ntk, device="cuda", dtype=torch.float64).t()
Cc = torch.zeros(ntk * nb, 2 * ntk, device="cuda", dtype=torch.float64).t()
Rr = torch.zeros(2 * ntk, ntk * nb, device="cuda", dtype=torch.float64).t()
Cm = torch.zeros(ntk * nb, ntk, device="cuda", dtype=torch.float64).t()
Rm = torch.zeros(ntk, ntk * nb, device="cuda", dtype=torch.float64).t()
ops.append(("dmma rule ntk=5", lambda: abft.abft_update_syrk(nb, ntk, L, cL, Cc, Rr, mL, Cm, Rm)))
for name, fn in ops:
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    print("done", name, flush=True)
