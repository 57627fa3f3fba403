"""Pins of the oracle's update rules and Alg. 2 driver (oracle/updates.py,
oracle/drivers.py) against independent facts: LAPACK's unblocked Cholesky
(numpy.linalg.cholesky) of the whole matrix, the checksum invariant
'maintained == recomputed' after every phase (L114, L149, L189), and fault
campaigns whose right answer is the fault-free factor.  CPU only."""
import numpy as np
import pytest

import synth_inputs as si
from oracle import checksum as ck
from oracle import drivers as dr
from oracle import updates as up


def _invariant(st, k, phase):
    """After each phase, every live checksum equals the recomputed one
    within tau (no flags) — checked on tiles whose checksums are maintained."""
    nt, nb = st.nt, st.nb
    tol = ck.Tol()
    if phase == "pd":
        tc = ck.check_tile(st, k, k, ck.LOWER, ck.COL, tol)
        assert not tc.Fc, (k, phase)
    elif phase == "pu":
        for I in range(k + 1, nt):
            tc = ck.check_tile(st, I, k, ck.GENERAL, ck.COL, tol)
            assert not tc.Fc, (k, phase, I)
    else:
        for I, J in ck.Tiles(k + 1, nt, k + 1, nt, True, ck.SYM_LOWER):
            tc = ck.check_tile(st, I, J, ck.SYM_LOWER if I == J else ck.GENERAL, ck.BOTH, tol)
            assert not tc.Fc and not tc.Fr, (k, phase, I, J)


@pytest.mark.parametrize("n,nb", [(256, 32), (512, 64), (384, 128)])
def test_ft_potrf_error_free_matches_lapack(n, nb):
    A = si.spd(n, seed=n + nb)
    L, stats = dr.ft_potrf(A, nb, invariant_hook=_invariant)
    Lref = np.linalg.cholesky(A)
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()
    assert stats.counts == [0] * 8 and stats.info == 0
    # Alg. 2 issues 2 checks per final iteration and 5 per other iteration
    nt = n // nb
    assert stats.n_checks == 5 * (nt - 1) + 2


def test_unprotected_driver_same_factor():
    A = si.spd(256, seed=3)
    L0, _ = dr.ft_potrf(A, 32, abft=False)
    L1, _ = dr.ft_potrf(A, 32, abft=True)
    assert np.abs(L0 - L1).max() <= 1e-13 * np.abs(L0).max()


def test_not_spd_reports_info():
    A = si.spd(128, seed=4)
    A[70, 70] = -1e6
    L, stats = dr.ft_potrf(A, 32, abft=False)
    assert stats.info == 64 + 7  # first failing minor, 1-based, inside tile 2


def _run(n, nb, injects, seed=0):
    A = si.spd(n, seed=seed)
    Lref, _ = dr.ft_potrf(A, nb)
    L, stats = dr.ft_potrf(A, nb, inject=injects)
    return A, Lref, L, stats


# one fault per run at every Alg. 2 hook, each expected to be fixed (paper
# Table VIII 'Y' outcomes for full checksums; readings c-8, c-11, c-25)
FIXABLE = [
    # (point, kind, gi, gj, bits)  at iteration k=2, n=256, nb=32
    (dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 70, 66, (61,)),   # DRAM in A_kk before the pre-PD check
    (dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 75, 75, (55, 52)),  # diagonal element
    (dr.AT_POST_PD, dr.KIND_PERSIST, 80, 70, (62,)),        # computation error in L_kk
    (dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 200, 70, (60,)),  # DRAM in the panel to be updated
    (dr.AT_POST_PU, dr.KIND_PERSIST, 150, 90, (63,)),       # computation error in L_ik
    (dr.AT_PRE_PU, dr.KIND_ONCHIP, 130, 68, (58,)),         # on-chip in PU update part -> 1D_ROW
    (dr.AT_PRE_TMU, dr.KIND_ONCHIP, 140, 72, (57,)),        # on-chip in TMU reference part -> 1D
    (dr.AT_PRE_TMU, dr.KIND_PERSIST, 170, 80, (54,)),       # DRAM in TMU reference part -> Fig. 4a
    (dr.AT_POST_TMU, dr.KIND_PERSIST, 230, 100, (59,)),     # computation error in the trailing matrix
    (dr.AT_POST_TMU, dr.KIND_PERSIST, 196, 196, (62,)),     # trailing diagonal element (SYRK output)
]


@pytest.mark.parametrize("case", range(len(FIXABLE)))
def test_fault_campaign_fixed(case):
    point, kind, gi, gj, bits = FIXABLE[case]
    inj = [dr.Inject(2, point, kind, 0, gi, gj, bits)]
    A, Lref, L, stats = _run(256, 32, inj)
    assert stats.uncorrectable == 0, stats.counts
    assert stats.counts[0] >= 1  # detected
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max(), np.abs(L - Lref).max()


def test_fig4a_repair_is_required():
    # without the repair the diagonal SYRK tile ends 2D (reading c-25)
    inj = [dr.Inject(2, dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 170, 80, (54,))]
    A = si.spd(256, seed=0)
    _, stats = dr.ft_potrf(A, 32, inject=inj, fig4a_repair=False)
    assert stats.uncorrectable >= 1
    _, stats = dr.ft_potrf(A, 32, inject=inj, fig4a_repair=True)
    assert stats.uncorrectable == 0 and stats.repairs_applied == 1


def test_fig4a_guard_huge_fault_detected_not_silent():
    # exponent flip to ~1e300 in a TMU reference element: the guarded repair
    # is skipped and the run ends DETECTED (R), never silently wrong (N)
    A = si.spd(256, seed=0)
    x = 0.3
    inj = [dr.Inject(2, dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 170, 80, (62,))]
    Lref, _ = dr.ft_potrf(A, 32)
    L, stats = dr.ft_potrf(A, 32, inject=inj)
    ok = np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()
    assert stats.repairs_skipped == 1
    assert ok or stats.uncorrectable >= 1


def test_pu_reference_fault_is_2d_and_restart_fixes_it():
    # on-chip flip in L_kk while PU reads it: every panel row is wrong -> 2D
    # (Table V); the local restart from the pre-PU copy (L430, f1) fixes it
    inj = [dr.Inject(2, dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 70, 66, (60,))]
    A = si.spd(256, seed=0)
    _, stats = dr.ft_potrf(A, 32, inject=inj, restart=False)
    assert stats.uncorrectable >= 1
    Lref, _ = dr.ft_potrf(A, 32)
    L, stats = dr.ft_potrf(A, 32, inject=inj)
    assert stats.uncorrectable == 0 and stats.restarts == 1
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()


@pytest.mark.parametrize("bit", [53, 57, 60, 63])
def test_pd_consumed_fault_restart(bit):
    # DRAM fault in A_kk between the pre-PD check and the PD: the PD consumes
    # it (2D in L_kk); the restart from the pre-PD copy gives the right factor
    inj = [dr.Inject(3, dr.AT_PRE_PD, dr.KIND_PERSIST, 0, 100, 99, (bit,))]
    A = si.spd(256, seed=1)
    Lref, _ = dr.ft_potrf(A, 32)
    L, stats = dr.ft_potrf(A, 32, inject=inj)
    assert stats.uncorrectable == 0 and stats.restarts == 1
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()


def test_checksum_memory_fault_repaired():
    inj = [dr.Inject(3, dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 1, 2 * 5 + 1, 100, (60,))]
    A, Lref, L, stats = _run(256, 32, inj)
    assert stats.uncorrectable == 0 and stats.counts[6] >= 1
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()


# ------------------------------------------------------------------- LU ----
import scipy.linalg as sla  # noqa: E402


def _lu_invariant(st, k, phase):
    nt = st.nt
    tol = ck.Tol()
    if phase == "pd":
        for I in range(k, nt):
            tc = ck.check_tile(st, I, k, ck.UNIT_LOWER if I == k else ck.GENERAL, ck.COL, tol)
            assert not tc.Fc, (k, phase, I)
        tc = ck.check_tile(st, k, k, ck.UPPER, ck.ROW, tol)
        assert not tc.Fr
        # trailing and left-panel checksums after the pivot swaps (c-14)
        for I, J in ck.Tiles(k + 1, nt, k + 1, nt):
            tc = ck.check_tile(st, I, J, ck.GENERAL, ck.BOTH, tol)
            assert not tc.Fc and not tc.Fr, (k, "swap", I, J)
        for I, J in ck.Tiles(0, nt, 0, k):
            if I >= J:
                tc = ck.check_tile(st, I, J, ck.UNIT_LOWER if I == J else ck.GENERAL, ck.COL, tol)
                assert not tc.Fc, (k, "swap-left", I, J)
    elif phase == "pu":
        for J in range(k + 1, nt):
            tc = ck.check_tile(st, k, J, ck.GENERAL, ck.ROW, tol)
            assert not tc.Fr, (k, phase, J)
    else:
        for I, J in ck.Tiles(k + 1, nt, k + 1, nt):
            tc = ck.check_tile(st, I, J, ck.GENERAL, ck.BOTH, tol)
            assert not tc.Fc and not tc.Fr, (k, phase, I, J)


@pytest.mark.parametrize("n,nb", [(256, 32), (512, 64), (384, 128)])
def test_ft_getrf_error_free_matches_lapack(n, nb):
    A = si.general(n, seed=n + nb)
    LU, piv, stats = dr.ft_getrf(A, nb, invariant_hook=_lu_invariant)
    lu, p = sla.lu_factor(A)
    assert np.array_equal(piv, p)
    assert np.abs(LU - lu).max() <= 1e-12 * np.abs(lu).max()
    assert stats.counts == [0] * 8


LU_FIXABLE = [
    (dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 100, 70, (61,)),   # DRAM in the column panel before PD
    (dr.AT_POST_PD, dr.KIND_PERSIST, 150, 80, (62,)),        # computation error in L21
    (dr.AT_POST_PD, dr.KIND_PERSIST, 66, 90, (58,)),         # computation error in U_kk
    (dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 70, 200, (60,)),   # DRAM in the row panel
    (dr.AT_POST_PU, dr.KIND_PERSIST, 75, 180, (63,)),        # computation error in U12
    (dr.AT_PRE_PU, dr.KIND_ONCHIP, 72, 130, (57,)),          # on-chip in PU update part -> 1D_COL
    (dr.AT_PRE_TMU, dr.KIND_ONCHIP, 140, 72, (57,)),         # on-chip in L21 during TMU -> 1D_ROW
    (dr.AT_PRE_TMU, dr.KIND_ONCHIP, 70, 140, (56,)),         # on-chip in U12 during TMU -> 1D_COL
    (dr.AT_PRE_TMU, dr.KIND_PERSIST, 170, 80, (54,)),        # DRAM in L21 -> Fig. 4a
    (dr.AT_PRE_TMU, dr.KIND_PERSIST, 80, 170, (55,)),        # DRAM in U12 -> Fig. 4a
    (dr.AT_POST_TMU, dr.KIND_PERSIST, 230, 100, (59,)),      # trailing computation error
]


@pytest.mark.parametrize("case", range(len(LU_FIXABLE)))
def test_lu_fault_campaign_fixed(case):
    point, kind, gi, gj, bits = LU_FIXABLE[case]
    A = si.general(256, seed=0)
    lu, p = sla.lu_factor(A)
    LU, piv, stats = dr.ft_getrf(A, 32, inject=[dr.Inject(2, point, kind, 0, gi, gj, bits)])
    assert stats.uncorrectable == 0, stats.counts
    assert stats.counts[0] >= 1
    assert np.array_equal(piv, p)
    assert np.abs(LU - lu).max() <= 1e-12 * np.abs(lu).max()


def test_lu_trailing_fault_in_a_pivot_row_fixed_before_the_swap():
    """A DRAM fault in a trailing row that the next panel's pivoting moves
    (row 70 = k·nb + 6 at k=2 is swapped unless it is its own pivot): the
    pre-swap row check (c-14b) must fix it before the swap deltas use it."""
    A = si.general(256, seed=0)
    lu, p = sla.lu_factor(A)
    assert p[70] != 70
    inj = [dr.Inject(1, dr.AT_POST_TMU, dr.KIND_PERSIST, 0, 70, 200, (60,))]
    LU, piv, stats = dr.ft_getrf(A, 32, inject=inj)
    assert stats.uncorrectable == 0 and stats.counts[5] >= 1
    assert any(c[1] == "pre_swap_rows" for c in stats.checks)
    assert np.array_equal(piv, p)
    assert np.abs(LU - lu).max() <= 1e-12 * np.abs(lu).max()


# ------------------------------------------------------------------- QR ----
def _qr_invariant(st, k, phase):
    nt = st.nt
    tol = ck.Tol()
    if phase == "pd":
        for I in range(k, nt):
            tc = ck.check_tile(st, I, k, ck.UNIT_LOWER if I == k else ck.GENERAL, ck.COL, tol)
            assert not tc.Fc, (k, phase, I)
        tc = ck.check_tile(st, k, k, ck.UPPER, ck.ROW, tol)
        assert not tc.Fr
        # below the diagonal tile, Q^T P [v1 v2] = 0 (Alg. 1 end state)
        n, nb = st.A.shape[0], st.nb
        below = st.rowchk[(k + 1) * nb:n, 2 * k:2 * k + 2]
        assert np.abs(below).max(initial=0) <= 1e-10 * max(1.0, np.abs(st.rowchk[k * nb:(k + 1) * nb, 2 * k]).max())
    else:
        for J in range(k + 1, nt):
            tc = ck.check_tile(st, k, J, ck.GENERAL, ck.ROW, tol)
            assert not tc.Fr, (k, "R12", J)
        for I, J in ck.Tiles(k + 1, nt, k + 1, nt):
            tc = ck.check_tile(st, I, J, ck.GENERAL, ck.BOTH, tol)
            assert not tc.Fc and not tc.Fr, (k, phase, I, J)


@pytest.mark.parametrize("n,nb", [(256, 32), (512, 64), (384, 128)])
def test_ft_geqrf_error_free_matches_lapack(n, nb):
    A = si.general(n, seed=n + nb + 1)
    H, tau, stats = dr.ft_geqrf(A, nb, invariant_hook=_qr_invariant)
    h, t = np.linalg.qr(A, mode="raw")  # LAPACK dgeqrf output (h transposed)
    h = h.T
    assert np.abs(H - h).max() <= 1e-12 * np.abs(h).max()
    assert np.abs(tau - t).max() <= 1e-12
    assert stats.counts == [0] * 8


def test_qr_last_column_convention():
    # dlarfg with x(2:) = 0 gives tau = 0 and R_nn = x_n (no sign flip, c-15)
    A = si.general(64, seed=3)
    H, tau, _ = dr.ft_geqrf(A, 32)
    h, t = np.linalg.qr(A, mode="raw")
    assert tau[-1] == 0.0 and t[-1] == 0.0 and H[-1, -1] == pytest.approx(h.T[-1, -1], rel=1e-12)


QR_FIXABLE = [
    (dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 100, 70, (61,)),   # DRAM in the column panel
    (dr.AT_POST_PD, dr.KIND_PERSIST, 150, 80, (62,)),        # computation error in V
    (dr.AT_POST_PD, dr.KIND_PERSIST, 66, 90, (58,)),         # computation error in R_kk
    (dr.AT_POST_TMU, dr.KIND_PERSIST, 230, 100, (59,)),      # trailing computation error
    (dr.AT_POST_TMU, dr.KIND_PERSIST, 70, 200, (60,)),       # R12 computation error
]


@pytest.mark.parametrize("case", range(len(QR_FIXABLE)))
def test_qr_fault_campaign_fixed(case):
    point, kind, gi, gj, bits = QR_FIXABLE[case]
    A = si.general(256, seed=0)
    h, t = np.linalg.qr(A, mode="raw")
    H, tau, stats = dr.ft_geqrf(A, 32, inject=[dr.Inject(2, point, kind, 0, gi, gj, bits)])
    assert stats.uncorrectable == 0, stats.counts
    assert stats.counts[0] >= 1
    assert np.abs(H - h.T).max() <= 1e-12 * np.abs(h).max()


def test_qr_tmu_reference_fault_detected():
    # DRAM fault in V consumed by the TMU: detected by the re-check, reported R
    A = si.general(256, seed=0)
    _, _, stats = dr.ft_geqrf(A, 32, inject=[dr.Inject(2, dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 170, 80, (54,))])
    assert stats.uncorrectable >= 1 and stats.repairs_skipped == 1


# ---- f1 local restart for LU and QR (L430) ---------------------------------
@pytest.mark.parametrize("bit,gi,gj", [(62, 200, 66), (60, 130, 70), (55, 64, 64)])
def test_lu_pd_consumed_fault_restart(bit, gi, gj):
    # a DRAM flip in the column panel between the pre-PD check and the PD is
    # consumed by getrf (2D, possibly other pivots); the restart takes back the
    # swaps outside the panel, restores the pre-PD copy and redoes the PD
    A = si.general(256, seed=31)
    ref, pref, _ = dr.ft_getrf(A, 64)
    inj = [dr.Inject(1, dr.AT_PRE_PD, dr.KIND_PERSIST, 0, gi, gj, (bit,))]
    _, _, s0 = dr.ft_getrf(A, 64, inject=inj, restart=False)
    assert s0.uncorrectable >= 1
    lu, piv, st = dr.ft_getrf(A, 64, inject=inj)
    assert st.uncorrectable == 0 and st.restarts == 1
    assert np.array_equal(piv, pref)
    assert np.abs(lu - ref).max() <= 1e-12 * np.abs(ref).max()


def test_lu_pd_undo_is_the_inverse_of_the_swaps():
    # lu_pd_undo after lu_pd_apply restores every row outside the panel and
    # the checksums (to rounding), whatever the pivots
    n, nb, k = 256, 32, 2
    st = ck.State.alloc(si.general(n, seed=32), nb)
    ck.encode(st, ck.Tiles(0, n // nb, 0, n // nb), ck.BOTH)
    before = st.copy()
    lu, piv, _, P0 = up.lu_panel_getrf(st, k)
    assert (piv != np.arange(k * nb, (k + 1) * nb)).sum() > 10
    up.lu_pd_apply(st, k, lu, piv, P0)
    up.lu_pd_undo(st, k, piv)
    out = np.r_[0:k * nb, (k + 1) * nb:n]
    assert np.array_equal(st.A[:, out], before.A[:, out])
    assert np.abs(st.colchk[:, out] - before.colchk[:, out]).max() <= 1e-12 * np.abs(before.colchk).max()
    assert np.array_equal(st.rowchk[:, 2 * (k + 1):], before.rowchk[:, 2 * (k + 1):])


def test_lu_pu_reference_fault_restart():
    # on-chip flip in L_kk while the PU reads it: U12 is 2D-wrong; restart
    A = si.general(256, seed=33)
    ref, _, _ = dr.ft_getrf(A, 32)
    inj = [dr.Inject(2, dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 70, 66, (60,))]
    _, _, s0 = dr.ft_getrf(A, 32, inject=inj, restart=False)
    assert s0.uncorrectable >= 1
    lu, _, st = dr.ft_getrf(A, 32, inject=inj)
    assert st.uncorrectable == 0 and st.restarts == 1
    assert np.abs(lu - ref).max() <= 1e-12 * np.abs(ref).max()


@pytest.mark.parametrize("bit,gi,gj", [(62, 200, 66), (57, 70, 70)])
def test_qr_pd_consumed_fault_restart(bit, gi, gj):
    A = si.general(256, seed=34)
    ref, tref, _ = dr.ft_geqrf(A, 64)
    inj = [dr.Inject(1, dr.AT_PRE_PD, dr.KIND_PERSIST, 0, gi, gj, (bit,))]
    _, _, s0 = dr.ft_geqrf(A, 64, inject=inj, restart=False)
    assert s0.uncorrectable >= 1
    qr, tau, st = dr.ft_geqrf(A, 64, inject=inj)
    assert st.uncorrectable == 0 and st.restarts == 1
    assert np.abs(qr - ref).max() <= 1e-12 * np.abs(ref).max() and np.abs(tau - tref).max() <= 1e-12


# ---- f1 Fig. 4b on-chip 1D detection and the periodic trailing check (L359) -
# Two on-chip faults in consecutive TMUs hit cached panel values of rows 197
# and 212 (both in tile row 6): each leaves a 1D row/column error across the
# trailing matrix; left alone they meet in tiles (6, 3..6) as a 2D error.
_ONCHIP_PAIR = [dr.Inject(1, dr.AT_PRE_TMU, dr.KIND_ONCHIP, 0, 197, 40, (55,)),
                dr.Inject(2, dr.AT_PRE_TMU, dr.KIND_ONCHIP, 0, 212, 67, (55,))]


def test_fig4b_stops_onchip_1d_errors_from_accumulating():
    A = si.spd(256, seed=41)
    Lref, _ = dr.ft_potrf(A, 32)
    _, s0 = dr.ft_potrf(A, 32, inject=_ONCHIP_PAIR, fig4b=False, restart=False)
    assert s0.uncorrectable >= 1
    L, st = dr.ft_potrf(A, 32, inject=_ONCHIP_PAIR, restart=False)
    assert st.uncorrectable == 0
    assert [c[1] for c in st.checks].count("fig4b") == 2
    assert any(f.cls in (ck.CLS_1D_ROW, ck.CLS_1D_COL) for f in st.fixes)
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()


def test_periodic_trailing_check_also_stops_the_accumulation():
    A = si.spd(256, seed=41)
    Lref, _ = dr.ft_potrf(A, 32)
    L, st = dr.ft_potrf(A, 32, inject=_ONCHIP_PAIR, fig4b=False, restart=False, trailing_check_period=1)
    assert st.uncorrectable == 0
    assert [c[1] for c in st.checks].count("periodic") == 256 // 32 - 1
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()


def test_fig4b_silent_without_faults():
    A = si.spd(256, seed=42)
    _, st = dr.ft_potrf(A, 32)
    assert "fig4b" not in [c[1] for c in st.checks]
    G = si.general(256, seed=43)
    _, _, st = dr.ft_getrf(G, 32, trailing_check_period=3)
    assert [c[1] for c in st.checks].count("periodic") == 2 and st.counts == [0] * 8


# ---------------------------------------------- checking schemes (c-34) --
# The four schemes the paper compares (L542, Table VIII; L343, L355): the new
# scheme (Alg. 2), full checksums with post-operation checks [13], column
# checksums with post-operation checks [51, 52], column checksums with
# prior-operation checks [11].
SCHEMES = [dr.SCHEME_NEW, dr.SCHEME_FULL_POST, dr.SCHEME_SINGLE_POST, dr.SCHEME_SINGLE_PRE]


@pytest.mark.parametrize("scheme", SCHEMES)
def test_scheme_error_free_matches_lapack(scheme):
    A = si.spd(256, seed=31)
    L, st = dr.ft_potrf(A, 32, scheme=scheme)
    Lref = np.linalg.cholesky(A)
    assert st.counts == [0] * 8 and not st.fixes
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()


# iteration-0 checks of each scheme: (phase, tile range, view, which), n=128 nb=32
SCHEME_CHECKS = {
    dr.SCHEME_NEW: [("pre_pd", 0, 1, 0, 1, ck.SYM_LOWER, ck.BOTH), ("post_pd", 0, 1, 0, 1, ck.LOWER, ck.COL),
                    ("pre_pu", 1, 4, 0, 1, ck.GENERAL, ck.BOTH), ("post_pu", 1, 4, 0, 1, ck.GENERAL, ck.COL),
                    ("post_tmu", 1, 4, 0, 1, ck.GENERAL, ck.COL)],
    dr.SCHEME_FULL_POST: [("post_pd", 0, 1, 0, 1, ck.LOWER, ck.COL), ("post_pu", 1, 4, 0, 1, ck.GENERAL, ck.COL),
                          ("post_tmu_trailing", 1, 4, 1, 4, ck.SYM_LOWER, ck.BOTH)],
    dr.SCHEME_SINGLE_POST: [("post_pd", 0, 1, 0, 1, ck.LOWER, ck.COL), ("post_pu", 1, 4, 0, 1, ck.GENERAL, ck.COL),
                            ("post_tmu_trailing", 1, 4, 1, 4, ck.SYM_LOWER, ck.COL)],
    dr.SCHEME_SINGLE_PRE: [("pre_pd", 0, 1, 0, 1, ck.SYM_LOWER, ck.COL), ("pre_pu", 1, 4, 0, 1, ck.GENERAL, ck.COL),
                           ("pre_tmu_panel", 1, 4, 0, 1, ck.GENERAL, ck.COL),
                           ("pre_tmu_trailing", 1, 4, 1, 4, ck.SYM_LOWER, ck.COL)],
}


@pytest.mark.parametrize("scheme", SCHEMES)
def test_scheme_check_sequence(scheme):
    """Each scheme checks what its definition says, in that order: inputs
    before the op (prior-operation, [11]), outputs after it (post-operation,
    [13], [51, 52]), or both for PD/PU plus the Fig. 4a panel re-check
    (Alg. 2).  Single-side schemes check column checksums only."""
    _, st = dr.ft_potrf(si.spd(128, seed=32), 32, scheme=scheme)
    got = [c[1:] for c in st.checks if c[0] == 0]
    assert got == SCHEME_CHECKS[scheme]


# (fault, outcome per scheme NEW / FULL_POST / SINGLE_POST / SINGLE_PRE) at n=256 nb=32,
# outcomes: Y = fixed (factor == LAPACK's within 1e-12), R = detected, uncorrectable
SCHEME_OUTCOMES = [
    # on-chip fault in a panel element during the TMU (L355): row AND column p of
    # the trailing matrix damaged (1D).  Full checksums fix 1D, single-side cannot
    # ("cannot tolerate errors causing 1D error propagation", L544)
    (dr.Inject(1, dr.AT_PRE_TMU, dr.KIND_ONCHIP, 0, 140, 40, (52,)), "YYRR"),
    # DRAM fault in A_kk between ops: a prior-operation check catches it before
    # the PD; a post-operation check finds the PD output inconsistent with the
    # copy taken after the fault -> 2D (L355: check before AND after PD)
    (dr.Inject(2, dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 0, 70, 66, (61,)), "YRRY"),
    # DRAM fault in the TMU reference part: only the Fig. 4a re-check + repair
    # (L357-L359) recovers it; the other schemes detect it (R)
    (dr.Inject(1, dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 140, 40, (52,)), "YRRR"),
    # 0D computation fault in the trailing matrix: every scheme fixes it
    (dr.Inject(1, dr.AT_POST_TMU, dr.KIND_PERSIST, 0, 200, 150, (60,)), "YYYY"),
]


@pytest.mark.parametrize("case", range(len(SCHEME_OUTCOMES)))
def test_scheme_outcomes(case):
    f, expect = SCHEME_OUTCOMES[case]
    A = si.spd(256, seed=3)
    Lref = np.linalg.cholesky(A)
    got = ""
    for scheme in SCHEMES:
        L, st = dr.ft_potrf(A, 32, inject=[f], scheme=scheme)
        ok = np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()
        got += "R" if st.uncorrectable else ("Y" if ok else "N")
    assert got == expect


# ---------------------------------------------- look-ahead (reading c-35) --
def test_lookahead_tmu_split_equals_full_tmu():
    """The TMU split by tile columns (column k+1, then the rest) is the same
    update as the whole TMU: data and every checksum / magnitude array."""
    n, nb, k = 256, 32, 1
    st = ck.State.alloc(si.spd(n, seed=51), nb)
    nt = n // nb
    ck.encode(st, ck.Tiles(0, nt, 0, nt, True, ck.SYM_LOWER))
    for kk in range(k + 1):  # factor panels 0..k so that panel k is an L panel
        up.chol_pd_rule(st, kk)
        up.chol_pu_data(st, kk)
        up.chol_pu_chk(st, kk)
        if kk < k:
            up.chol_tmu_data(st, kk)
            up.chol_tmu_chk(st, kk)
    a, b = st.copy(), st.copy()
    up.chol_tmu_data(a, k)
    up.chol_tmu_chk(a, k)
    r1, c2 = (k + 1) * nb, (k + 2) * nb
    for c0, c1 in ((r1, c2), (c2, n)):
        up.chol_tmu_data(b, k, c0, c1)
        up.chol_tmu_chk(b, k, c0, c1)
    for x, y in ((a.A, b.A), (a.colchk, b.colchk), (a.rowchk, b.rowchk), (a.colmag, b.colmag), (a.rowmag, b.rowmag)):
        assert np.abs(x - y).max() <= 1e-13 * max(1.0, np.abs(x).max())


@pytest.mark.parametrize("p", [70, 100, 200])
def test_lookahead_restricted_repairs_add_up_to_the_full_repair(p):
    """Reading c-35: the Fig. 4a repair restricted to tile column k+1 plus the
    one restricted to the columns after it is the unrestricted repair."""
    n, nb, k = 256, 32, 1
    st = ck.State.alloc(si.spd(n, seed=52), nb)
    nt = n // nb
    ck.encode(st, ck.Tiles(0, nt, 0, nt, True, ck.SYM_LOWER))
    q = k * nb + 5
    before, after = 0.25, 0.75
    a, b = st.copy(), st.copy()
    assert up.chol_fig4a_repair(a, k, p, q, before, after) == "applied"
    r1, c2 = (k + 1) * nb, (k + 2) * nb
    up.chol_fig4a_repair(b, k, p, q, before, after, r1, c2)
    up.chol_fig4a_repair(b, k, p, q, before, after, c2, n)
    for x, y in ((a.A, b.A), (a.colchk, b.colchk), (a.rowchk, b.rowchk), (a.colmag, b.colmag), (a.rowmag, b.rowmag)):
        assert np.array_equal(x, y)


@pytest.mark.parametrize("n,nb", [(256, 32), (384, 128)])
def test_lookahead_error_free(n, nb):
    A = si.spd(n, seed=n + 7)
    L, stats = dr.ft_potrf(A, nb, lookahead=True, invariant_hook=_invariant)
    Lref = np.linalg.cholesky(A)
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()
    nt = n // nb
    assert stats.counts == [0] * 8 and stats.n_checks == 6 * (nt - 1) + 2  # one extra re-check per iteration


@pytest.mark.parametrize("case", range(len(FIXABLE)))
def test_lookahead_fault_outcomes_equal_alg2(case):
    """Same faults with and without look-ahead: the same factor, fixes
    (positions, classes) and counters (the predicate keeps Alg. 2's order
    around every fault hook)."""
    point, kind, gi, gj, bits = FIXABLE[case]
    inj = [dr.Inject(2, point, kind, 0, gi, gj, bits)]
    A = si.spd(256, seed=0)
    L0, s0 = dr.ft_potrf(A, 32, inject=inj)
    L1, s1 = dr.ft_potrf(A, 32, inject=inj, lookahead=True)
    assert s1.counts == s0.counts and s1.restarts == s0.restarts and s1.repairs_applied == s0.repairs_applied
    assert sorted((f.gi, f.gj, f.cls, f.kind) for f in s1.fixes) == sorted((f.gi, f.gj, f.cls, f.kind) for f in s0.fixes)
    assert np.abs(L1 - L0).max() <= 1e-13 * np.abs(L0).max()


def test_lu_lookahead_tmu_split_and_restricted_repairs():
    """LU (c-35): the TMU split by tile columns equals the whole TMU, and the
    two restricted Fig. 4a repairs add up to the unrestricted one (an L21 and
    a U12 element)."""
    n, nb, k = 256, 32, 1
    st = ck.State.alloc(si.general(n, seed=61), nb)
    nt = n // nb
    ck.encode(st, ck.Tiles(0, nt, 0, nt), ck.BOTH)
    for kk in range(k + 1):
        up.lu_pd(st, kk)
        up.lu_pu_data(st, kk)
        up.lu_pu_chk(st, kk)
        if kk < k:
            up.lu_tmu_data(st, kk)
            up.lu_tmu_chk(st, kk)
    r1, c2 = (k + 1) * nb, (k + 2) * nb
    a, b = st.copy(), st.copy()
    up.lu_tmu_data(a, k)
    up.lu_tmu_chk(a, k)
    for c0, c1 in ((r1, c2), (c2, n)):
        up.lu_tmu_data(b, k, c0, c1)
        up.lu_tmu_chk(b, k, c0, c1)
    for x, y in ((a.A, b.A), (a.colchk, b.colchk), (a.rowchk, b.rowchk), (a.colmag, b.colmag), (a.rowmag, b.rowmag)):
        assert np.abs(x - y).max() <= 1e-13 * max(1.0, np.abs(x).max())
    for gi, gj in ((150, k * nb + 4), (k * nb + 6, 150), (k * nb + 6, r1 + 3)):
        a, b = st.copy(), st.copy()
        assert up.lu_fig4a_repair(a, k, gi, gj, 0.25, 0.75) == "applied"
        up.lu_fig4a_repair(b, k, gi, gj, 0.25, 0.75, r1, c2)
        up.lu_fig4a_repair(b, k, gi, gj, 0.25, 0.75, c2, n)
        for x, y in ((a.A, b.A), (a.colchk, b.colchk), (a.rowchk, b.rowchk), (a.colmag, b.colmag),
                     (a.rowmag, b.rowmag)):
            assert np.array_equal(x, y), (gi, gj)


@pytest.mark.parametrize("n,nb", [(256, 32), (384, 128)])
def test_lu_lookahead_error_free(n, nb):
    A = si.general(n, seed=n + 9)
    LU, piv, st = dr.ft_getrf(A, nb, lookahead=True, invariant_hook=_lu_invariant)
    lu, p = sla.lu_factor(A)
    assert np.array_equal(piv, p) and np.abs(LU - lu).max() <= 1e-12 * np.abs(lu).max()
    _, _, s0 = dr.ft_getrf(A, nb)
    assert st.counts == [0] * 8 and st.n_checks == s0.n_checks + 2 * (n // nb - 1)  # both panels re-checked twice


@pytest.mark.parametrize("case", range(len(LU_FIXABLE)))
def test_lu_lookahead_fault_outcomes_equal_alg2(case):
    point, kind, gi, gj, bits = LU_FIXABLE[case]
    inj = [dr.Inject(2, point, kind, 0, gi, gj, bits)]
    A = si.general(256, seed=0)
    L0, p0, s0 = dr.ft_getrf(A, 32, inject=inj)
    L1, p1, s1 = dr.ft_getrf(A, 32, inject=inj, lookahead=True)
    assert s1.counts == s0.counts and s1.restarts == s0.restarts and s1.repairs_applied == s0.repairs_applied
    assert sorted((f.gi, f.gj, f.cls, f.kind) for f in s1.fixes) == sorted((f.gi, f.gj, f.cls, f.kind) for f in s0.fixes)
    assert np.array_equal(p0, p1) and np.abs(L1 - L0).max() <= 1e-13 * np.abs(L0).max()


@pytest.mark.parametrize("bit,gi,gj", [(62, 200, 66), (60, 130, 70), (55, 64, 64)])
def test_lu_lookahead_split_pd_restart_equals_alg2(bit, gi, gj):
    """A PD-consumed fault in a panel the look-ahead factored (split PD, c-35):
    the restart redoes only the part inside the panel (nothing outside moved
    yet) and ends at Alg. 2's result: same pivots, factor, counters, fixes."""
    A = si.general(256, seed=31)
    inj = [dr.Inject(1, dr.AT_PRE_PD, dr.KIND_PERSIST, 0, gi, gj, (bit,))]
    l0, p0, s0 = dr.ft_getrf(A, 64, inject=inj)
    l1, p1, s1 = dr.ft_getrf(A, 64, inject=inj, lookahead=True)
    assert s1.restarts == s0.restarts == 1 and s1.uncorrectable == s0.uncorrectable == 0
    assert s1.counts == s0.counts
    assert np.array_equal(p1, p0) and np.abs(l1 - l0).max() <= 1e-13 * np.abs(l0).max()
