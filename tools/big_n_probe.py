"""Per-rep encode / verify bandwidth at a large n with NVML power, SM/memory
clock and throttle reasons sampled between reps (why do n=65536 sweep points
vary?).  python tools/big_n_probe.py N NB BITS REPS"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import pynvml
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

n, nb, bits, reps = (int(x) for x in sys.argv[1:5])
dt = torch.float64 if bits == 64 else torch.float32
pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
A = si.general_device(n, seed=n, dtype=dt)
mat = abft.Mat.alloc(A, nb, mags=False)
rep = abft.Report.alloc(mat)
tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
t = abft.tiles(0, n // nb, 0, n // nb)
by = n * n * A.element_size() * (1 + 4 / nb)
for i in range(reps):
    for name, fn in (("enc", lambda: abft.abft_encode(mat, t)),
                     ("ver", lambda: abft.abft_verify(mat, t, abft.BOTH, tol, rep))):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b)
        p = pynvml.nvmlDeviceGetPowerUsage(h) / 1000
        sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
        mem = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_MEM)
        rs = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
        print(f"rep {i:2d} {name} {ms:7.3f} ms {by / ms / 1e6:7.0f} GB/s  power {p:6.0f} W  sm {sm} MHz  mem {mem} MHz"
              f"  reasons 0x{rs:x}", flush=True)
