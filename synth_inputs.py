"""Seeded synthetic input generators shared by the oracle tests, the GPU
parity tests and bench.py.

This module holds NONE of the method's arithmetic (no checksums, no
thresholds, no factorizations): it only draws matrices and fault plans from
seeded generators, following the input recipe of DESIGN.md §3:

* general (LU, QR, bandwidth sweep): A_ij ~ U(-1, 1);
* SPD (Cholesky): A = (M + M^T)/2 + n*I with M ~ U(-1, 1);
* integer tiles (exact-sum pins): A_ij uniform integers in [-R, R];
* bit-flip plans (paper §X.A): element positions and XOR masks.

Host arrays are numpy, float64 unless a dtype is given; `*_device` variants
draw on the GPU with a seeded torch generator so the multi-GiB bench inputs
never touch the host.  Semantics are mathematical (A[i, j] = row i, column
j); the binding is responsible for the column-major layout of the C ABI.
"""
from __future__ import annotations

import numpy as np


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def general(m: int, n: int | None = None, seed: int = 0, dtype=np.float64) -> np.ndarray:
    """U(-1,1) general matrix (SURVEY §8d 'general')."""
    n = m if n is None else n
    return rng(seed).uniform(-1.0, 1.0, size=(m, n)).astype(dtype)


def spd(n: int, seed: int = 0, dtype=np.float64) -> np.ndarray:
    """(M + M^T)/2 + n*I, M ~ U(-1,1): diagonally dominant SPD."""
    M = rng(seed).uniform(-1.0, 1.0, size=(n, n))
    S = (M + M.T) * 0.5
    S[np.diag_indices(n)] += n
    return S.astype(dtype)


def stieltjes(n: int, seed: int = 0, dtype=np.float64) -> np.ndarray:
    """n*I - B with B symmetric, B_ij ~ U(0,1) off the diagonal, B_ii = 0:
    a diagonally dominant SPD matrix with non-positive off-diagonal entries
    (a Stieltjes matrix).  Used by the magnitude pins: its Cholesky factor
    keeps one sign pattern, so the absolute-value computation has no
    cancellation off the diagonal."""
    M = rng(seed).uniform(0.0, 1.0, size=(n, n))
    B = (M + M.T) * 0.5
    B[np.diag_indices(n)] = 0.0
    S = -B
    S[np.diag_indices(n)] = float(n)
    return S.astype(dtype)


def m_matrix(n: int, seed: int = 0, dtype=np.float64) -> np.ndarray:
    """n*I - B with B_ij ~ U(0,1) off the diagonal (B_ii = 0): a
    column-diagonally-dominant nonsingular M-matrix (partial pivoting never
    swaps; L and U keep non-positive off-diagonal entries).  Magnitude pins
    for LU, like `stieltjes` for Cholesky."""
    B = rng(seed).uniform(0.0, 1.0, size=(n, n))
    B[np.diag_indices(n)] = 0.0
    S = -B
    S[np.diag_indices(n)] = float(n)
    return S.astype(dtype)


def integers(m: int, n: int | None = None, seed: int = 0, R: int = 64, dtype=np.float64) -> np.ndarray:
    """Integer-valued matrix in [-R, R]; every checksum of it is an exactly
    representable integer, so sums are bit-exact in any order."""
    n = m if n is None else n
    return rng(seed).integers(-R, R + 1, size=(m, n)).astype(dtype)


def flip_bits(value: float, bits, dtype=np.float64) -> float:
    """XOR the given bit positions of one IEEE value (the paper's XOR fault,
    L540).  Pure bit manipulation, no arithmetic of the method."""
    if dtype == np.float64:
        u = np.array([value], dtype=np.float64).view(np.uint64)
        mask = np.uint64(0)
        for b in bits:
            mask |= np.uint64(1) << np.uint64(b)
        return float((u ^ mask).view(np.float64)[0])
    u = np.array([value], dtype=np.float32).view(np.uint32)
    mask = np.uint32(0)
    for b in bits:
        mask |= np.uint32(1) << np.uint32(b)
    return float((u ^ mask).view(np.float32)[0])


def mask_of(bits) -> int:
    m = 0
    for b in bits:
        m |= 1 << int(b)
    return m


def random_positions(n_tiles_r: int, n_tiles_c: int, nb: int, seed: int, lower_only: bool = False):
    """One random (local i, local j) per tile: the config-1 'one flip per
    tile' plan (BASELINE configs[0], paper L275 single-fault assumption)."""
    g = rng(seed)
    out = []
    for J in range(n_tiles_c):
        for I in range(n_tiles_r):
            if lower_only and I < J:
                continue
            out.append((I, J, int(g.integers(0, nb)), int(g.integers(0, nb))))
    return out


# ---------------------------------------------------------------- device --
def general_device(m: int, n: int | None = None, seed: int = 0, dtype=None, device="cuda"):
    """Column-major U(-1,1) matrix drawn on the GPU (bench-sized inputs)."""
    import torch

    n = m if n is None else n
    dtype = dtype or torch.float64
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    # storage (n, m) row-major == (m, n) column-major
    buf = torch.rand((n, m), generator=g, dtype=dtype, device=device)
    buf.mul_(2.0).sub_(1.0)
    return buf.t()


def spd_device(n: int, seed: int = 0, dtype=None, device="cuda"):
    """(M + M^T)/2 + n*I with M ~ U(-1,1), drawn on the GPU; symmetric, so the
    returned column-major view is the same matrix."""
    import torch

    dtype = dtype or torch.float64
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    buf = torch.rand((n, n), generator=g, dtype=dtype, device=device)
    buf.mul_(2.0).sub_(1.0)
    S = buf + buf.t()
    del buf
    S.mul_(0.5)
    S.diagonal().add_(float(n))
    return S.t()


def spd_block_cyclic_device(n: int, nb: int, P: int, Q: int, rank: int, seed: int = 0, dtype=None, device="cuda"):
    """This rank's tiles of the SPD matrix S = (M + M^T)/2 + n*I under the 2D
    block-cyclic layout (tile (I, J) on rank (I mod P)*Q + J mod Q), as one
    column-major local matrix.  Tile M_IJ ~ U(-1,1) is drawn from its own
    seed (seed, I, J), so every rank builds its tiles without the full
    matrix; the distribution is the one of `spd`/`spd_device`."""
    import torch

    dtype = dtype or torch.float64
    nt = n // nb
    p, q = divmod(rank, Q)
    rows, cols = list(range(p, nt, P)), list(range(q, nt, Q))
    buf = torch.empty((len(cols) * nb, len(rows) * nb), dtype=dtype, device=device)  # col-major storage
    g = torch.Generator(device=device)

    def tile(I, J):
        g.manual_seed(seed * 1_000_003 + I * nt + J)
        return torch.rand((nb, nb), generator=g, dtype=dtype, device=device).mul_(2.0).sub_(1.0)

    for jl, J in enumerate(cols):
        for il, I in enumerate(rows):
            S = tile(I, J)
            S.add_(tile(J, I).t()).mul_(0.5)
            if I == J:
                S.diagonal().add_(float(n))
            buf[jl * nb:(jl + 1) * nb, il * nb:(il + 1) * nb] = S.t()
    return buf.t()
