"""Panel-check latency vs slab split (ABFT_NSLAB forces the split; one
process per value): verify (COL) of a k-tile panel column, n=30720 nb=512
fp64, graph-captured back-to-back launches, warm L2 like the driver's checks.
  for s in 0 1 2 4 8; do ABFT_NSLAB=$s python tools/slab_tune.py; done"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft


def timed(fn, reps=50):
    """Device time per call (us): calls captured in a CUDA graph."""
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


n, nb = 30720, 512
nt = n // nb
A = si.spd_device(n, seed=3)
mat = abft.Mat.alloc(A, nb)
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
abft.abft_encode(mat, abft.tiles(0, nt, 0, nt))
torch.cuda.synchronize()
res = {"nslab": int(os.environ.get("ABFT_NSLAB", "0"))}
for k in (1, 2, 4, 8, 12, 16, 20, 24, 30, 37, 40, 48, 59):
    tl = abft.tiles(nt - k, nt, nt - k - 1, nt - k)
    us = timed(lambda: abft.abft_verify(mat, tl, abft.COL, tol, rep))
    res[k] = us
    print(f"nslab={res['nslab']} tiles={k:3d} verify {us:7.2f} us  {k * nb * nb * 8 / us / 1e3:7.0f} GB/s", flush=True)
os.makedirs("gpurun_out", exist_ok=True)
with open(f"gpurun_out/slab_tune_{res['nslab']}.json", "w") as f:
    json.dump(res, f)
