"""Probe: how does the diagonal-tile Cholesky scale with the tile size on B200
(cuSOLVER via torch), and what would a 2-level recursive split cost?"""
import torch

torch.backends.cuda.preferred_linalg_library("cusolver")


def spd(n):
    g = torch.randn(n, n, dtype=torch.float64, device="cuda")
    return g @ g.T + n * torch.eye(n, dtype=torch.float64, device="cuda")


def t(fn, reps=50):
    for _ in range(5):
        fn()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps * 1e3


for n in (32, 64, 128, 256, 512, 1024):
    A = spd(n)
    print(f"cholesky n={n}: {t(lambda: torch.linalg.cholesky(A)):.1f} us", flush=True)


def rec(A, leaf):
    n = A.shape[0]
    if n <= leaf:
        return torch.linalg.cholesky(A)
    h = n // 2
    L11 = rec(A[:h, :h], leaf)
    L21 = torch.linalg.solve_triangular(L11, A[h:, :h].T, upper=False).T
    L22 = rec(A[h:, h:] - L21 @ L21.T, leaf)
    L = torch.zeros_like(A)
    L[:h, :h] = L11
    L[h:, :h] = L21
    L[h:, h:] = L22
    return L


A = spd(512)
for leaf in (64, 128, 256):
    err = (rec(A, leaf) - torch.linalg.cholesky(A)).abs().max().item()
    print(f"recursive 512 leaf={leaf}: {t(lambda: rec(A, leaf)):.1f} us (err {err:.1e})", flush=True)
