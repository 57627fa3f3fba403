"""Latency of the checksum pass on small tile sets (the driver's per-iteration
checks): CUDA-event average over many back-to-back launches, warm L2."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb = int(os.environ.get('SP_N', 30720)), 512
nt = n // nb
A = si.spd_device(n, seed=3)
mat = abft.Mat.alloc(A, nb)
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
abft.abft_encode(mat, abft.tiles(0, nt, 0, nt))
fixes = torch.zeros(64 * abft.FIX_BYTES, dtype=torch.uint8, device="cuda")
nfx = torch.zeros(1, dtype=torch.int32, device="cuda")
torch.cuda.synchronize()


def t(fn, reps=50):
    """Device time per call: the calls are captured in a CUDA graph so host
    (ctypes) overhead does not leave gaps on the timeline."""
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(5):
            fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(reps):
            fn()
    g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(4):
        g.replay()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / (4 * reps) * 1e3


for name, tl, which in [
    ("1 tile GENERAL both", abft.tiles(5, 6, 5, 6), abft.BOTH),
    ("1 tile SYM_LOWER both", abft.tiles(5, 6, 5, 6, False, abft.SYM_LOWER), abft.BOTH),
    ("1 tile LOWER col", abft.tiles(5, 6, 5, 6, False, abft.LOWER), abft.COL),
    ("8 tiles panel col", abft.tiles(nt - 8, nt, 4, 5), abft.COL),
    ("nt-1 tiles panel both", abft.tiles(1, nt, 0, 1), abft.BOTH),
    ("nt-1 tiles panel col", abft.tiles(1, nt, 0, 1), abft.COL),
    ("30 tiles panel col", abft.tiles(nt - 30, nt, nt - 31, nt - 30), abft.COL),
]:
    if tl.I1 > nt or tl.J1 > nt or tl.I0 < 0 or tl.J0 < 0:
        continue
    us_e = t(lambda: abft.abft_encode(mat, tl, which))
    us_v = t(lambda: abft.abft_verify(mat, tl, which, tol, rep))
    us_l = t(lambda: abft.abft_locate_correct(mat, tl, which, tol, rep, fixes, nfx))
    ntile = (tl.I1 - tl.I0) * (tl.J1 - tl.J0)
    gbs = ntile * nb * nb * 8 * (1 + 4 / nb) / (us_v * 1e-6) / 1e9
    print(f"n={n} {name:24s} verify {us_v:8.2f} us ({gbs:7.0f} GB/s)  encode {us_e:8.2f} us  locate {us_l:6.2f} us",
          flush=True)
