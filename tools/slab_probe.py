"""Encode / verify GB/s of one full-matrix pass (GENERAL view) for slab-count
experiments: ABFT_NSLAB=s python tools/slab_probe.py N NB f64|f32"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb = int(sys.argv[1]), int(sys.argv[2])
dt, es = (torch.float64, 8) if sys.argv[3] == "f64" else (torch.float32, 4)
A = si.general_device(n, seed=n, dtype=dt)
mat = abft.Mat.alloc(A, nb, mags=False)
t = abft.tiles(0, n // nb, 0, n // nb)
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
L2 = torch.cuda.get_device_properties(0).L2_cache_size
flush = torch.empty(4 * L2, dtype=torch.uint8, device="cuda")
evict = torch.empty(4 * L2 // 8, dtype=torch.float64, device="cuda")


def timed(fn, reps=20):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        flush.add_(1)  # write a buffer larger than L2, then read another (clean L2)
        evict.sum()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


gb = n * n * es * (1 + 4 / nb) / 1e9
te = timed(lambda: abft.abft_encode(mat, t, abft.BOTH))
tv = timed(lambda: abft.abft_verify(mat, t, abft.BOTH, tol, rep))
print(f"nslab={os.environ.get('ABFT_NSLAB', 'auto')} n={n} nb={nb} {sys.argv[3]}: encode {gb / te:.2f} TB/s "
      f"verify {gb / tv:.2f} TB/s", flush=True)
