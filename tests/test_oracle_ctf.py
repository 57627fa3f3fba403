"""Pins of the QR CTF check (row f2; L263) in oracle/updates.py and its use
in oracle/drivers.ft_geqrf, against facts outside the oracle: LAPACK dgeqrf's
reflectors, the explicit product of the Householder matrices
H_j = I − τ_j v_j v_j^T, orthogonality of Q, and the fault-free factor.
CPU only."""
import numpy as np
import pytest
import scipy.linalg as sla

import synth_inputs as si
from oracle import drivers as dr
from oracle import updates as up


def _panel(m, nb, seed):
    P = si.general(m, nb, seed=seed)
    qr, tau, _, info = sla.lapack.dgeqrf(P)
    assert info == 0
    V = np.tril(qr, -1)[:, :nb]
    V[:nb, :nb] += np.eye(nb)
    return P, qr, V, tau


@pytest.mark.parametrize("m,nb", [(64, 16), (512, 64), (1024, 128)])
def test_ctf_is_the_product_of_the_reflectors(m, nb):
    P, qr, V, tau = _panel(m, nb, seed=m)
    T = up.qr_T(V, tau)
    Q = np.eye(m)
    for j in range(nb):  # brute force: Q = H_0 H_1 ... H_{nb-1}
        v = V[:, j]
        Q = Q @ (np.eye(m) - tau[j] * np.outer(v, v))
    assert np.abs(Q - (np.eye(m) - V @ T @ V.T)).max() <= 1e-13
    assert np.abs(Q.T @ Q - np.eye(m)).max() <= 1e-13
    R = np.triu(qr[:nb, :nb])
    assert np.abs(Q[:, :nb] @ R - P).max() <= 1e-13 * np.abs(P).max() * nb
    assert up.qr_ctf_check(V, T)[0] == 0


def test_ctf_check_flags_every_significant_flip():
    P, qr, V, tau = _panel(512, 32, seed=3)
    T = up.qr_T(V, tau)
    rng = np.random.default_rng(4)
    for _ in range(200):
        i, j = rng.integers(0, 32, size=2)
        bit = int(rng.integers(40, 63))
        Tb = T.copy()
        Tb[i, j] = si.flip_bits(Tb[i, j], [bit])
        if Tb[i, j] == T[i, j] or abs(Tb[i, j] - T[i, j]) < 1e-3 * max(1.0, abs(T[i, j])):
            continue  # flips of a zero's low bits are below any threshold
        assert up.qr_ctf_check(V, Tb)[0] > 0, (i, j, bit)


def test_ctf_check_flags_a_t_of_another_panel():
    _, _, V, tau = _panel(256, 32, seed=5)
    _, _, V2, tau2 = _panel(256, 32, seed=6)
    assert up.qr_ctf_check(V, up.qr_T(V2, tau2))[0] > 0


def test_zero_tau_column_passes():
    # a column already zero below the diagonal: LAPACK returns tau = 0 (H = I)
    P = si.general(128, 16, seed=7)
    P[1:, 0] = 0.0
    qr, tau, _, _ = sla.lapack.dgeqrf(P)
    assert tau[0] == 0.0
    V = np.tril(qr, -1)[:, :16]
    V[:16, :16] += np.eye(16)
    assert up.qr_ctf_check(V, up.qr_T(V, tau))[0] == 0


def test_geqrf_driver_recomputes_a_corrupted_t():
    n, nb = 256, 64
    A = si.general(n, seed=8)
    ref, tref, s0 = dr.ft_geqrf(A, nb)
    assert s0.ctf_flagged == 0
    inj = [dr.Inject(1, dr.AT_POST_PD, dr.KIND_PERSIST, 3, 5, 9, (61,))]
    out, tau, st = dr.ft_geqrf(A, nb, inject=inj)
    assert (st.ctf_flagged, st.ctf_recomputed, st.uncorrectable) == (1, 1, 0)
    assert np.abs(out - ref).max() <= 1e-12 * np.abs(ref).max()
    # without the check the corrupted T reaches the trailing update
    bad, _, _ = dr.ft_geqrf(A, nb, abft=False, inject=inj)
    assert not np.abs(bad - ref).max() <= 1e-6
