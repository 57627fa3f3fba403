"""GPU parity of the checksum update rules (§8 rows a4–a6) against the
oracle's rules (oracle/updates.py) and, for the generic ops, against the
triangular-solve / matmul definitions."""
import numpy as np
import pytest
import torch

import synth_inputs as si
from oracle import checksum as ck
from oracle import updates as up
from tests.gpu_helpers import dev, gpu_state_to_oracle, host

pytestmark = pytest.mark.gpu


def _tri(nb, seed, lower=True, unit=False):
    g = si.rng(seed)
    T = g.uniform(-1, 1, (nb, nb)) / nb
    T = np.tril(T) if lower else np.triu(T)
    np.fill_diagonal(T, 1.0 if unit else g.uniform(1, 2, nb))
    return T


# tile sizes from 32 to 1024, checksum-vector counts from 6 to the 118 of a
# 60-tile panel
@pytest.mark.parametrize("nb,nvec", [(64, 10), (512, 118), (1024, 6), (32, 10)])
@pytest.mark.parametrize("side,uplo,trans,diag", [("R", "L", "T", "N"), ("L", "L", "N", "U"), ("L", "U", "N", "N"),
                                                  ("R", "U", "N", "N"), ("R", "L", "N", "N"), ("L", "U", "T", "N")])
def test_update_trsm_matches_solve(lib, side, uplo, trans, diag, nb, nvec):
    T = _tri(nb, 1, uplo == "L", diag == "U")
    shape = (nvec, nb) if side == "R" else (nb, nvec)
    X = si.general(*shape, seed=2)
    M = np.abs(si.general(*((nvec // 2, nb) if side == "R" else (nb, nvec // 2)), seed=3))
    Td, Xd, Md = dev(T), dev(X), dev(M)
    lib.abft_update_trsm(side, uplo, trans, diag, nb, Td, Xd, nvec, Md, nvec // 2)
    torch.cuda.synchronize()
    opT = T.T if trans == "T" else T
    Tinv = np.linalg.inv(opT)
    ref = X @ Tinv if side == "R" else Tinv @ X
    mref = M @ np.abs(Tinv) if side == "R" else np.abs(Tinv) @ M
    assert np.abs(host(Xd) - ref).max() <= 1e-12 * np.abs(ref).max()
    assert np.abs(host(Md) - mref).max() <= 1e-12 * np.abs(mref).max()


@pytest.mark.parametrize("side,trans", [("R", "T"), ("L", "N")])
def test_update_trsm_f32(lib, side, trans):
    nb, nvec = 512, 40
    T = _tri(nb, 4, True, False).astype(np.float32)
    shape = (nvec, nb) if side == "R" else (nb, nvec)
    X = si.general(*shape, seed=5).astype(np.float32)
    Td, Xd = dev(T, torch.float32), dev(X, torch.float32)
    lib.abft_update_trsm(side, "L", trans, "N", nb, Td, Xd, nvec)
    torch.cuda.synchronize()
    opT = T.astype(np.float64).T if trans == "T" else T.astype(np.float64)
    Tinv = np.linalg.inv(opT)
    ref = X @ Tinv if side == "R" else Tinv @ X
    assert np.abs(host(Xd) - ref).max() <= 1e-4 * np.abs(ref).max()


# padded leading dimensions (the drivers' checksum arrays: ld = 2 nt > nvec)
# and every vector-block tail (nvec not a multiple of the kernel's 16)
@pytest.mark.parametrize("prec", ["f64", "f32"])
@pytest.mark.parametrize("side,trans,nb,nvec", [("R", "T", 512, 37), ("L", "N", 256, 3), ("R", "N", 128, 17),
                                                ("L", "T", 64, 33)])
def test_update_trsm_inv_padded(lib, prec, side, trans, nb, nvec):
    dt = torch.float64 if prec == "f64" else torch.float32
    T = _tri(nb, 6, True, False)
    if prec == "f32":
        T = T.astype(np.float32).astype(np.float64)
    W = np.linalg.inv(T)
    shape = (nvec, nb) if side == "R" else (nb, nvec)
    X = si.general(*shape, seed=7)
    M = np.abs(si.general(*((nvec // 2 + 1, nb) if side == "R" else (nb, nvec // 2 + 1)), seed=8))
    if prec == "f32":
        W, X, M = (a.astype(np.float32).astype(np.float64) for a in (W, X, M))
    Wd = dev(W, dt, ld=nb + 3)
    Xd = dev(X, dt, ld=shape[0] + 5)
    Md = dev(M, dt, ld=M.shape[0] + 2)
    lib.abft_update_trsm_inv(side, trans, Wd, Xd, nvec, Md, M.shape[1] if side == "L" else M.shape[0])
    torch.cuda.synchronize()
    opW = W.T if trans == "T" else W
    ref = X @ opW if side == "R" else opW @ X
    mref = M @ np.abs(opW) if side == "R" else np.abs(opW) @ M
    tol = 1e-12 if prec == "f64" else 1e-5
    assert np.abs(host(Xd) - ref).max() <= tol * np.abs(ref).max()
    assert np.abs(host(Md) - mref).max() <= tol * np.abs(mref).max()


# fp64 runs the DMMA rule kernel (abft_rule_dmma.cu, mode 1): a small case, a
# ragged one (N, K off the 32 / 16 tiles), and a 60-tile LU panel's rule
@pytest.mark.parametrize("M2,N,K", [(12, 96, 32), (6, 75, 40), (118, 2000, 512)])
@pytest.mark.parametrize("which,tX,tY", [(1, "N", "T"), (2, "T", "N"), (1, "N", "N"), (2, "N", "N"), (1, "T", "N"),
                                         (2, "N", "T"), (1, "T", "T"), (2, "T", "T")])
def test_update_gemm_matches_matmul(lib, which, tX, tY, M2, N, K):
    X = si.general(*((M2, K) if (which == 1) == (tX == "N") else (K, M2)), seed=4)
    Y = si.general(*((K, N) if (which == 1) == (tY == "N") else (N, K)), seed=5)
    C = si.general(*((M2, N) if which == 1 else (N, M2)), seed=6)
    Xm = np.abs(si.general(*((M2 // 2, K) if (which == 1) == (tX == "N") else (K, M2 // 2)), seed=7))
    Cm = np.abs(si.general(*((M2 // 2, N) if which == 1 else (N, M2 // 2)), seed=8))
    d = [dev(a) for a in (X, Y, C, Xm, Cm)]
    lib.abft_update_gemm(which, tX, tY, -1.0, d[0], d[1], d[2], M2, N, K, d[3], d[4])
    torch.cuda.synchronize()
    opX = X.T if tX == "T" else X
    opY = Y.T if tY == "T" else Y
    opXm = Xm.T if tX == "T" else Xm
    ref = C - (opX @ opY if which == 1 else opY @ opX)
    mref = Cm + (opXm @ np.abs(opY) if which == 1 else np.abs(opY) @ opXm)
    assert np.abs(host(d[2]) - ref).max() <= 1e-12 * np.abs(ref).max()
    assert np.abs(host(d[4]) - mref).max() <= 1e-12 * np.abs(mref).max()


def _chol_state(n, nb):
    A = si.spd(n, seed=n)
    st = ck.State.alloc(A, nb)
    ck.encode(st, ck.Tiles(0, n // nb, 0, n // nb, True, ck.SYM_LOWER))
    return st


def test_panel_potrf_matches_oracle_rule(lib):
    n, nb = 512, 128
    st = _chol_state(n, nb)
    mat = lib.Mat(dev(st.A), nb, dev(st.colchk), dev(st.rowchk), dev(st.colmag), dev(st.rowmag))
    diag = lib.Mat(mat.A[:nb, :nb], nb, mat.colchk[0:2, 0:nb], None, mat.colmag[0:1, 0:nb], None)
    info = torch.zeros(1, dtype=torch.int32, device="cuda")
    Linv = lib.colmajor_empty(nb, nb)
    lib.abft_panel_potrf(diag, info, Linv)
    torch.cuda.synchronize()
    assert info.item() == 0
    up.chol_pd_rule(st, 0)
    g = gpu_state_to_oracle(mat)
    L = np.tril(st.A[:nb, :nb])
    assert np.abs(np.tril(g.A[:nb, :nb]) - L).max() <= 1e-13 * np.abs(L).max()
    assert np.abs(g.colchk[0:2, :nb] - st.colchk[0:2, :nb]).max() <= 1e-12 * np.abs(st.colchk[0:2, :nb]).max()
    assert np.abs(g.colmag[0, :nb] - st.colmag[0, :nb]).max() <= 1e-12 * np.abs(st.colmag[0, :nb]).max()
    assert np.abs(host(Linv) - np.linalg.inv(L)).max() <= 1e-12 * np.abs(np.linalg.inv(L)).max()


# fp64 runs the fused DMMA kernel (abft_rule_dmma.cu): one 192-row chunk of
# checksum rows (768/128), two chunks (2240/32: 69 tile rows -> 216 rows),
# the metric's nb (2048/512), a later iteration, and nb=16 (cuBLAS route)
@pytest.mark.parametrize("n,nb,k", [(768, 128, 0), (2240, 32, 0), (2048, 512, 0), (1536, 256, 2), (512, 16, 1)])
@pytest.mark.parametrize("rows", [True, False])
def test_update_syrk_matches_oracle_rule(lib, n, nb, k, rows):
    st = _chol_state(n, nb)
    up.chol_pd_rule(st, k)
    up.chol_pu_data(st, k)
    up.chol_pu_chk(st, k)
    mat = lib.Mat(dev(st.A), nb, dev(st.colchk), dev(st.rowchk), dev(st.colmag), dev(st.rowmag))
    row_before = host(mat.rowchk).copy(), host(mat.rowmag).copy()
    up.chol_tmu_chk(st, k)  # the oracle's checksum step of the TMU
    r1, ntk = (k + 1) * nb, n // nb - k - 1
    k2, k1 = 2 * (k + 1), k + 1
    lib.abft_update_syrk(nb, ntk, mat.A[r1:, k * nb:r1], mat.colchk[k2:, k * nb:r1], mat.colchk[k2:, r1:],
                         mat.rowchk[r1:, k2:] if rows else None, mat.colmag[k1:, k * nb:r1], mat.colmag[k1:, r1:],
                         mat.rowmag[r1:, k1:] if rows else None)
    torch.cuda.synchronize()
    g = gpu_state_to_oracle(mat)
    for I, J in ck.Tiles(k + 1, n // nb, k + 1, n // nb, True):
        cs, rs = slice(J * nb, (J + 1) * nb), slice(I * nb, (I + 1) * nb)
        pairs = [(g.colchk[2 * I:2 * I + 2, cs], st.colchk[2 * I:2 * I + 2, cs]), (g.colmag[I, cs], st.colmag[I, cs])]
        if rows:
            pairs += [(g.rowchk[rs, 2 * J:2 * J + 2], st.rowchk[rs, 2 * J:2 * J + 2]),
                      (g.rowmag[rs, J], st.rowmag[rs, J])]
        for a, b in pairs:
            assert np.abs(a - b).max() <= 1e-12 * max(np.abs(b).max(), 1.0), (I, J)
    if not rows:  # the single-checksum call leaves the row side alone
        assert np.array_equal(host(mat.rowchk), row_before[0]) and np.array_equal(host(mat.rowmag), row_before[1])


@pytest.mark.parametrize("nb", [32, 64, 128, 512, 1024])
@pytest.mark.parametrize("uplo,diag", [("L", "N"), ("U", "N"), ("L", "U"), ("U", "U")])
def test_tri_inverse_matches_numpy(lib, nb, uplo, diag):
    T = _tri(nb, nb, uplo == "L", diag == "U")
    junk = si.general(nb, seed=9)  # the other triangle must be ignored
    Tfull = T + (np.triu(junk, 1) if uplo == "L" else np.tril(junk, -1))
    if diag == "U":
        np.fill_diagonal(Tfull, 7.0)  # ignored for a unit diagonal
    Td = dev(Tfull)
    W = lib.colmajor_zeros(nb, nb)
    W.fill_(3.0)
    lib.abft_tri_inverse(uplo, diag, Td, W)
    torch.cuda.synchronize()
    ref = np.linalg.inv(T)
    assert np.abs(host(W) - ref).max() <= 1e-12 * np.abs(ref).max()
