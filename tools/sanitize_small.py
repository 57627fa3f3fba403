"""Tiny workloads for compute-sanitizer (racecheck / synccheck / memcheck)
of the pass (encode / verify, every launch shape: RECT, SEG, DIAG, slabbed
tiles) and locate kernels, plus one small ft_potrf with faults (gated
restart, Fig. 4a repair, look-ahead side stream, the DMMA TMU rule kernel,
the panel row rule).
  compute-sanitizer --tool racecheck python tools/sanitize_small.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

torch.cuda.set_device(0)
for dt in (torch.float64, torch.float32):
    for nb, n, view, lower in ((32, 256, abft.SYM_LOWER, True), (64, 256, abft.GENERAL, False),
                               (512, 1024, abft.GENERAL, False), (256, 768, abft.LOWER, True)):
        A = abft.to_colmajor(torch.from_numpy(si.spd(n, seed=nb)).to(dt).cuda())
        mat = abft.Mat.alloc(A, nb)
        t = abft.tiles(0, n // nb, 0, n // nb, lower, view)
        abft.abft_encode(mat, t)
        mat.A[5, 3] += 100.0  # one flagged tile
        rep = abft.Report.alloc(mat)
        tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0)
        abft.abft_verify(mat, t, abft.BOTH, tol, rep)
        fixbuf = torch.zeros(256 * abft.FIX_BYTES, dtype=torch.uint8, device="cuda")
        nfix = torch.zeros(1, dtype=torch.int32, device="cuda")
        abft.abft_locate_correct(mat, t, abft.BOTH, tol, rep, fixbuf, nfix)
        sub = abft.tiles(1, n // nb, 0, 1)  # a sub-range: slabbed single-column launch
        abft.abft_verify(mat, sub, abft.COL, tol, rep)
        torch.cuda.synchronize()
        print(dt, nb, n, "fixes", int(nfix.item()), "counts", rep.counts.tolist(), flush=True)
ctx = abft.Context()
A = abft.to_colmajor(torch.from_numpy(si.spd(1024, seed=3)).cuda())
inj = [(2, abft.AT_PRE_PU, abft.KIND_ONCHIP, 0, 300, 270, 1 << 60),     # L_kk read by the PU: 2D, gated restart
       (4, abft.AT_POST_TMU, abft.KIND_PERSIST, 0, 900, 700, 1 << 59)]  # trailing 0D fix
rc, info, st = abft.ft_potrf(ctx, A, 128, inject=inj)
torch.cuda.synchronize()
print("ft_potrf rc", rc, "restarts", st.restarts, "fixes", st.n_fixes, flush=True)
