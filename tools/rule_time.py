"""Time the Cholesky TMU checksum rule (abft_update_syrk) at the trailing
sizes of an n=30720, nb=512 factorization.  fp64 takes the fused DMMA
kernel; ABFT_RULE_CUBLAS=1 selects the GEMM route.  Usage:
  [ABFT_RULE_CUBLAS=1] python tools/rule_time.py [NB] [NTK ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_sc_chenlllwtolzgc18_b200 import abft

nb = int(sys.argv[1]) if len(sys.argv) > 1 else 512
ntks = [int(x) for x in sys.argv[2:]] or [59, 45, 30, 15, 5, 1]
route = "cublas" if os.environ.get("ABFT_RULE_CUBLAS") else "dmma"
for ntk in ntks:
    nk = ntk * nb
    g = torch.Generator(device="cuda").manual_seed(ntk)
    L = torch.randn(nb, nk, device="cuda", dtype=torch.float64, generator=g).t()  # column-major nk x nb
    cL = torch.randn(nb, 2 * ntk, device="cuda", dtype=torch.float64, generator=g).t()
    mL = torch.rand(nb, ntk, device="cuda", dtype=torch.float64, generator=g).t()
    Cc = torch.zeros(nk, 2 * ntk, device="cuda", dtype=torch.float64).t()
    Rr = torch.zeros(2 * ntk, nk, device="cuda", dtype=torch.float64).t()
    Cm = torch.zeros(nk, ntk, device="cuda", dtype=torch.float64).t()
    Rm = torch.zeros(ntk, nk, device="cuda", dtype=torch.float64).t()
    run = lambda: abft.abft_update_syrk(nb, ntk, L, cL, Cc, Rr, mL, Cm, Rm)
    for _ in range(3):
        run()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 20
    a.record()
    for _ in range(reps):
        run()
    b.record()
    torch.cuda.synchronize()
    us = a.elapsed_time(b) / reps * 1e3
    flops = 2.0 * 3 * ntk * nk * nb
    print(f"{route} nb={nb} ntk={ntk}: {us:.1f} us  {flops / us / 1e6:.1f} TF/s", flush=True)

