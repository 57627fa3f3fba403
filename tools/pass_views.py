"""Encode / verify time of one range under different diagonal views (is the
masked diagonal path a bottleneck of lower-only passes?).
  python tools/pass_views.py N NB BITS"""
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
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
nt = n // nb


def timed(fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return sorted(ts)[reps // 2]


for name, t in [("full GENERAL", abft.tiles(0, nt, 0, nt)),
                ("lower GENERAL diag", abft.tiles(0, nt, 0, nt, True, abft.GENERAL)),
                ("lower SYM_LOWER diag", abft.tiles(0, nt, 0, nt, True, abft.SYM_LOWER)),
                ("lower LOWER diag", abft.tiles(0, nt, 0, nt, True, abft.LOWER)),
                ("lower UPPER diag", abft.tiles(0, nt, 0, nt, True, abft.UPPER)),
                ("diag only SYM", None)]:
    if t is None:
        continue
    ntiles = nt * nt if not t.lower_only else nt * (nt + 1) // 2
    by = ntiles * nb * nb * A.element_size()
    te = timed(lambda: abft.abft_encode(mat, t))
    tv = timed(lambda: abft.abft_verify(mat, t, abft.BOTH, tol, rep))
    print(f"n={n} nb={nb} fp{bits} {name:22s} encode {by / te / 1e6:7.0f} GB/s  verify {by / tv / 1e6:7.0f} GB/s")
