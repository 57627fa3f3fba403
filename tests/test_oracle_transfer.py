"""Pins of oracle/transfer.py (Alg. 2 lines 3-7 with the PD on the host,
L364-L372; reading c-28) and of the oracle drivers' pd_location="host" mode,
against facts independent of the oracle's arithmetic: exact integer sums,
the original value of a flipped element, the unflipped factor.  CPU only."""
import numpy as np
import pytest

import synth_inputs as si
from oracle import checksum as ck
from oracle import drivers as dr
from oracle import transfer as tr


def test_guard_is_the_definition_on_integers():
    # integer panel: every sum is exact, so the guard equals brute force
    nb, P = 8, si.integers(24, 8, seed=1, R=100)
    G = tr.transfer_guard(P, nb)
    for I in range(3):
        for j in range(8):
            assert G[2 * I, j] == sum(P[I * nb + i, j] for i in range(nb))
            assert G[2 * I + 1, j] == sum((i + 1) * P[I * nb + i, j] for i in range(nb))


@pytest.mark.parametrize("bit", [30, 52, 62])
def test_host_check_locates_every_single_flip(bit):
    nb = 8
    P0 = si.general(16, 8, seed=bit)
    G = tr.transfer_guard(P0, nb)
    for gi in range(16):
        for j in range(8):
            P = P0.copy()
            P[gi, j] = si.flip_bits(P[gi, j], [bit])
            fl, fixes, ok = tr.host_check(P, G, nb)
            assert ok and fl == 1 and len(fixes) == 1, (gi, j)
            assert fixes[0][:2] == (gi, j)
            assert abs(P[gi, j] - P0[gi, j]) <= 1e-14 * np.abs(P0[:, j]).sum()


def test_host_check_clean_panel_is_silent():
    P = si.general(64, 32, seed=3)
    G = tr.transfer_guard(P, 32)
    assert tr.host_check(P.copy(), G, 32) == (0, [], True)


def test_host_check_two_flips_in_a_column_need_a_retransfer():
    P0 = si.general(16, 8, seed=5)
    G = tr.transfer_guard(P0, 8)
    P = P0.copy()
    P[1, 3] += 1.0
    P[5, 3] -= 2.0  # ratio 10 > nb: no single-error pattern explains it
    assert not tr.host_check(P, G, 8)[2]


def test_host_check_corrupted_guard_entry_needs_a_retransfer():
    P = si.general(16, 8, seed=6)
    G = tr.transfer_guard(P, 8)
    G[2, 4] = si.flip_bits(G[2, 4], [60])  # e-entry of tile 1, column 4
    fl, fixes, ok = tr.host_check(P.copy(), G, 8)
    assert fl == 1 and not fixes and not ok


def test_host_check_non_finite_is_located_by_the_fallback():
    P0 = si.general(16, 8, seed=7)
    G = tr.transfer_guard(P0, 8)
    for bad in (np.inf, np.nan, 1e308):
        P = P0.copy()
        P[3, 2] = bad
        fl, fixes, ok = tr.host_check(P, G, 8)
        assert ok and [f[:2] for f in fixes] == [(3, 2)]
        assert abs(P[3, 2] - P0[3, 2]) <= 1e-14 * np.abs(P0[:, 2]).sum()
    P = P0.copy()
    P[3, 2], P[4, 2] = np.inf, np.inf  # two non-finite: no candidate survives
    assert not tr.host_check(P, G, 8)[2]


def test_device_check_single_flip_and_2d():
    P0 = si.general(32, 16, seed=8)
    G = tr.transfer_guard(P0, 16)
    P = P0.copy()
    P[20, 5] = si.flip_bits(P[20, 5], [61])
    fl, fixes, unc = tr.device_check(P, G, 16)
    assert fl == 1 and unc == 0 and [(f.gi, f.gj) for f in fixes] == [(20, 5)]
    assert np.abs(P - P0).max() <= 1e-14 * np.abs(P0).max()
    P = P0.copy()
    P[17, 2] += 5.0
    P[19, 2] += 7.0
    P[18, 9] += 1.0
    P[21, 11] += 2.0
    assert tr.device_check(P, G, 16)[2] == 1


def _inj(k, point, gi, gj, bits=(62,)):
    return dr.Inject(k, point, dr.KIND_PERSIST, 0, gi, gj, tuple(bits))


def test_host_mode_fault_free_equals_device_mode():
    A = si.spd(256, seed=11)
    L0, s0 = dr.ft_potrf(A, 32)
    L1, s1 = dr.ft_potrf(A, 32, pd_location="host")
    assert np.abs(L1 - L0).max() <= 1e-14 * np.abs(L0).max()
    assert s1.counts == [0] * 8 and s1.xfer == tr.XferStats()
    G = si.general(256, seed=12)
    lu0, p0, _ = dr.ft_getrf(G, 64)
    lu1, p1, s = dr.ft_getrf(G, 64, pd_location="host")
    assert (p0 == p1).all() and np.abs(lu1 - lu0).max() <= 1e-13 * np.abs(lu0).max()
    assert s.xfer == tr.XferStats()
    qr0, t0, _ = dr.ft_geqrf(G, 64)
    qr1, t1, s = dr.ft_geqrf(G, 64, pd_location="host")
    assert np.abs(qr1 - qr0).max() <= 1e-13 * np.abs(qr0).max() and np.abs(t1 - t0).max() <= 1e-14
    assert s.xfer == tr.XferStats()


def test_host_mode_potrf_transfer_faults_fixed():
    n, nb = 256, 32
    A = si.spd(n, seed=13)
    Lref = np.linalg.cholesky(A)
    inj = [_inj(2, dr.AT_D2H, 2 * nb + 5, 2 * nb + 3),      # host copy of A_22
           _inj(4, dr.AT_H2D, 4 * nb + 9, 4 * nb + 1),      # factored L_44 on arrival
           _inj(5, dr.AT_D2H, 5 * nb + 1, 5 * nb + 0),      # two flips in one column:
           _inj(5, dr.AT_D2H, 5 * nb + 7, 5 * nb + 0, (61,))]  # -> re-transfer
    L, st = dr.ft_potrf(A, nb, inject=inj, pd_location="host")
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()
    x = st.xfer
    assert (x.d2h_fixed, x.retransfers, x.h2d_fixed, x.uncorrectable) == (1, 1, 1, 0)
    assert st.uncorrectable == 0
    assert [(f.gi, f.gj) for f in x.fixes] == [(4 * nb + 9, 4 * nb + 1)]


def test_host_mode_lu_qr_transfer_faults_fixed():
    n, nb = 256, 64
    G = si.general(n, seed=14)
    lu0, p0, _ = dr.ft_getrf(G, nb)
    inj = [_inj(1, dr.AT_D2H, 200, nb + 7), _inj(2, dr.AT_H2D, 2 * nb + 40, 2 * nb + 3)]
    lu1, p1, st = dr.ft_getrf(G, nb, inject=inj, pd_location="host")
    assert (p0 == p1).all() and np.abs(lu1 - lu0).max() <= 1e-12 * np.abs(lu0).max()
    assert (st.xfer.d2h_fixed, st.xfer.h2d_fixed, st.uncorrectable) == (1, 1, 0)
    qr0, t0, _ = dr.ft_geqrf(G, nb)
    inj = [_inj(0, dr.AT_D2H, 100, 5), _inj(1, dr.AT_H2D, nb + 3, nb + 60)]
    qr1, t1, st = dr.ft_geqrf(G, nb, inject=inj, pd_location="host")
    assert np.abs(qr1 - qr0).max() <= 1e-12 * np.abs(qr0).max() and np.abs(t1 - t0).max() <= 1e-12
    assert (st.xfer.d2h_fixed, st.xfer.h2d_fixed, st.uncorrectable) == (1, 1, 0)


def test_host_mode_unprotected_transfer_fault_is_silent():
    # without the guard a D2H flip is consumed by the host PD: the factor is wrong
    A = si.spd(128, seed=15)
    L, _ = dr.ft_potrf(A, 32, abft=False, inject=[_inj(1, dr.AT_D2H, 40, 33, (52,))],
                        pd_location="host")
    assert not np.abs(L - np.linalg.cholesky(A)).max() <= 1e-6
