"""Pins of the oracle's magnitude checksums (reading c-6) and of the verify
`refresh` (DESIGN §4 c-6), against facts the mathematics fixes rather than
against the oracle's own update code.  CPU only.

The threshold is tau_e = 2*gamma_nb*m (L124-L133: the a-priori bound
gamma_n*||A||*||B|| of one update, carried per component).  m is the column
(row) sum of the running absolute-value computation: every op of the
decomposition applied with |.| on its operands and its subtractions turned
into additions.  Two facts hold whatever the input:

* lower bound: m >= e^T|X| (triangle inequality), after every phase;
* no cancellation, no slack: when every product the decomposition forms has
  the sign of the value it updates, |.| of the computation IS the
  computation, so m == e^T|X| exactly (to rounding).  A Stieltjes matrix
  (SPD, non-positive off-diagonals) for Cholesky and a column-dominant
  M-matrix for LU have that property everywhere except on the diagonal
  elements, whose slack is a closed form of LAPACK's factor:
  2*sum_q L[g,q]^2 (Cholesky), 2*sum_q L[g,q]*U[q,g] (LU).
* QR: the first Householder vector of a panel has no cancellation either
  (x1 - beta has the sign of x1), so right after a refreshed pre-PD check
  m_c(V_I)[first column] == e^T|V_I[:, 0]| with V from LAPACK's dgeqrf.

The expected values come from numpy.linalg.cholesky / scipy.linalg.lu /
numpy.linalg.qr(mode='raw') and the original matrix — never from the
oracle's state.
"""
import numpy as np
import pytest
import scipy.linalg as sla

import synth_inputs as si
from oracle import checksum as ck
from oracle import drivers as dr
from oracle import updates as up

RTOL = 1e-11
NO_REFRESH = ck.Tol(refresh=False)


def _colsum(X):
    return np.abs(X).sum(axis=0)


def _rowsum(X):
    return np.abs(X).sum(axis=1)


def _close(got, want, what):
    err = np.abs(got - want).max() / max(np.abs(want).max(), 1e-300)
    assert err <= RTOL, (what, err)


def _lower_bounds(st, tiles_views, which):
    """m >= e^T|X| (columns) and m >= |X|e (rows) on the listed tiles."""
    nb = st.nb
    slack = 1e-12
    for I, J, view in tiles_views:
        X = ck.tile_view(st.A, I, J, nb, view)
        if which & ck.COL:
            m = st.colmag[I, J * nb:(J + 1) * nb]
            assert np.all(m >= _colsum(X) * (1 - slack)), ("col", I, J, (m / _colsum(X).clip(1e-300)).min())
        if which & ck.ROW:
            m = st.rowmag[I * nb:(I + 1) * nb, J]
            assert np.all(m >= _rowsum(X) * (1 - slack)), ("row", I, J, (m / _rowsum(X).clip(1e-300)).min())


# --------------------------------------------------------------- Cholesky --
@pytest.mark.parametrize("n,nb", [(256, 32), (384, 64)])
def test_cholesky_magnitudes_closed_form_stieltjes(n, nb):
    A = si.stieltjes(n, seed=n + nb)
    L = np.linalg.cholesky(A)
    assert np.all(np.tril(L, -1) <= 0)  # the sign pattern the closed form needs
    nt = n // nb
    seen = set()

    def hook(st, k, phase):
        r1 = (k + 1) * nb
        seen.add(phase)
        if phase == "pu":
            for I in range(k + 1, nt):
                rows = slice(I * nb, (I + 1) * nb)
                _close(st.colmag[I, k * nb:r1], _colsum(L[rows, k * nb:r1]), ("pu", k, I))
        elif phase == "tmu":
            # trailing matrix after k+1 updates, from LAPACK's factor
            S = A - L[:, :r1] @ L[:, :r1].T
            slack = 2.0 * (L[:, :r1] ** 2).sum(axis=1)  # the diagonal's |.| slack
            for I in range(k + 1, nt):
                for J in range(k + 1, I + 1):
                    rs, cs = slice(I * nb, (I + 1) * nb), slice(J * nb, (J + 1) * nb)
                    X = S[rs, cs]
                    mc, mr = _colsum(X), _rowsum(X)
                    if I == J:
                        mc = mc + slack[cs]
                        mr = mr + slack[rs]
                    _close(st.colmag[I, cs], mc, ("tmu col", k, I, J))
                    _close(st.rowmag[rs, J], mr, ("tmu row", k, I, J))

    Lo, stats = dr.ft_potrf(A, nb, tol=NO_REFRESH, invariant_hook=hook)
    assert stats.counts == [0] * 8
    assert {"pu", "tmu"} <= seen
    assert np.abs(Lo - L).max() <= 1e-12 * np.abs(L).max()


def test_cholesky_pu_magnitude_rule_brute_force_inverse():
    """m_c(L_ik) = m_c(A_ik)*|L_kk^{-T}| with the inverse from np.linalg.inv."""
    n, nb, k = 256, 32, 2
    st = ck.State.alloc(si.spd(n, seed=7), nb)
    st.colmag[:] = si.rng(8).uniform(0.5, 2.0, size=st.colmag.shape)
    s = slice(k * nb, (k + 1) * nb)
    st.A[s, s] = np.linalg.cholesky(st.A[s, s])
    before = st.colmag[k + 1:, s].copy()
    up.chol_pu_chk(st, k)
    Linv = np.linalg.inv(np.tril(st.A[s, s]))
    _close(st.colmag[k + 1:, s], before @ np.abs(Linv.T), "pu rule")


@pytest.mark.parametrize("n,nb", [(256, 32)])
def test_cholesky_magnitude_lower_bound_every_phase(n, nb):
    A = si.spd(n, seed=11)
    nt = n // nb

    def hook(st, k, phase):
        if phase == "pd":
            _lower_bounds(st, [(k, k, ck.LOWER)], ck.COL)
        elif phase == "pu":
            _lower_bounds(st, [(I, k, ck.GENERAL) for I in range(k + 1, nt)], ck.COL)
        else:
            tv = [(I, J, ck.SYM_LOWER if I == J else ck.GENERAL) for I, J in ck.Tiles(k + 1, nt, k + 1, nt, True)]
            _lower_bounds(st, tv, ck.BOTH)

    for tol in (NO_REFRESH, ck.Tol(refresh=True)):
        dr.ft_potrf(A, nb, tol=tol, invariant_hook=hook)


# --------------------------------------------------------------------- LU --
@pytest.mark.parametrize("n,nb", [(256, 32), (384, 64)])
def test_lu_magnitudes_closed_form_m_matrix(n, nb):
    A = si.m_matrix(n, seed=n + nb)
    P, Lr, Ur = sla.lu(A)
    assert np.array_equal(P, np.eye(n))  # column dominance: no pivoting
    assert np.all(np.tril(Lr, -1) <= 0) and np.all(np.triu(Ur, 1) <= 0)
    nt = n // nb
    seen = set()

    def hook(st, k, phase):
        r0, r1 = k * nb, (k + 1) * nb
        seen.add(phase)
        if phase == "pd":
            for I in range(k + 1, nt):
                rows = slice(I * nb, (I + 1) * nb)
                _close(st.colmag[I, r0:r1], _colsum(Lr[rows, r0:r1]), ("pd L", k, I))
        elif phase == "pu":
            for J in range(k + 1, nt):
                cs = slice(J * nb, (J + 1) * nb)
                _close(st.rowmag[r0:r1, J], _rowsum(Ur[r0:r1, cs]), ("pu U", k, J))
        else:
            S = A - Lr[:, :r1] @ Ur[:r1, :]
            slack = 2.0 * np.einsum("gq,qg->g", Lr[:, :r1], Ur[:r1, :])
            for I in range(k + 1, nt):
                for J in range(k + 1, nt):
                    rs, cs = slice(I * nb, (I + 1) * nb), slice(J * nb, (J + 1) * nb)
                    X = S[rs, cs]
                    mc, mr = _colsum(X), _rowsum(X)
                    if I == J:
                        mc = mc + slack[cs]
                        mr = mr + slack[rs]
                    _close(st.colmag[I, cs], mc, ("tmu col", k, I, J))
                    _close(st.rowmag[rs, J], mr, ("tmu row", k, I, J))

    LU, piv, stats = dr.ft_getrf(A, nb, tol=NO_REFRESH, invariant_hook=hook)
    assert stats.counts == [0] * 8 and np.array_equal(piv, np.arange(n))
    assert {"pd", "pu", "tmu"} <= seen


def test_lu_swap_rule_moves_magnitudes_with_the_rows():
    """After any sequence of row exchanges applied with the c-14 rule to a
    freshly encoded state, the magnitudes are those of the permuted matrix:
    colmag == e^T|X|, rowmag == |X|e (the rule moves |x| exactly)."""
    n, nb = 256, 32
    st = ck.State.alloc(si.general(n, seed=21), nb)
    nt = n // nb
    ck.encode(st, ck.Tiles(0, nt, 0, nt), ck.BOTH)
    g = si.rng(22)
    cols = np.arange(n)
    for _ in range(40):
        p, q = (int(x) for x in g.integers(0, n, size=2))
        if p == q:
            continue
        up.lu_swap_rule(st, p, q, cols, st.A[p].copy(), st.A[q].copy(), row_chk_cols=range(nt))
        st.A[[p, q]] = st.A[[q, p]]
    for I, J in ck.Tiles(0, nt, 0, nt):
        rs, cs = slice(I * nb, (I + 1) * nb), slice(J * nb, (J + 1) * nb)
        _close(st.colmag[I, cs], _colsum(st.A[rs, cs]), ("col", I, J))
        _close(st.rowmag[rs, J], _rowsum(st.A[rs, cs]), ("row", I, J))


def test_lu_magnitude_lower_bound_every_phase():
    n, nb = 256, 32
    A = si.general(n, seed=12)
    nt = n // nb

    def hook(st, k, phase):
        if phase == "pd":
            tv = [(I, k, ck.UNIT_LOWER if I == k else ck.GENERAL) for I in range(k, nt)]
            _lower_bounds(st, tv, ck.COL)
            _lower_bounds(st, [(k, k, ck.UPPER)], ck.ROW)
        elif phase == "pu":
            _lower_bounds(st, [(k, J, ck.GENERAL) for J in range(k + 1, nt)], ck.ROW)
        else:
            _lower_bounds(st, [(I, J, ck.GENERAL) for I, J in ck.Tiles(k + 1, nt, k + 1, nt)], ck.BOTH)

    for tol in (NO_REFRESH, ck.Tol(refresh=True)):
        dr.ft_getrf(A, nb, tol=tol, invariant_hook=hook)


# --------------------------------------------------------------------- QR --
@pytest.mark.parametrize("n,nb,k", [(256, 32, 0), (256, 32, 3), (384, 64, 1)])
def test_qr_first_reflector_magnitude_closed_form(n, nb, k):
    """Alg. 1 on panel k of a freshly encoded matrix (m_c = e^T|P|): the
    first reflector's magnitude per tile equals e^T|V_I[:, 0]| of LAPACK's
    dgeqrf of that panel."""
    A = si.general(n, seed=n + nb + 5)
    nt = n // nb
    r0 = k * nb
    h, _ = np.linalg.qr(A[r0:, r0:r0 + nb], mode="raw")
    V = np.tril(h.T, -1) + np.eye(n - r0, nb)  # LAPACK's unit lower reflectors
    st = ck.State.alloc(A, nb)
    ck.encode(st, ck.Tiles(0, nt, 0, nt), ck.BOTH)
    up.qr_pd_alg1(st, k)
    for I in range(k, nt):
        rows = slice((I - k) * nb, (I - k + 1) * nb)
        _close(st.colmag[I, r0], _colsum(V[rows, 0:1])[0], ("m_v", k, I))
    # the driver's first panel sees the same fresh magnitudes (no refresh needed)
    seen = []

    def hook(st, kk, phase):
        if phase == "pd" and kk == 0:
            h0, _ = np.linalg.qr(A[:, :nb], mode="raw")
            V0 = np.tril(h0.T, -1) + np.eye(n, nb)
            for I in range(nt):
                _close(st.colmag[I, 0], _colsum(V0[I * nb:(I + 1) * nb, 0:1])[0], ("driver m_v", I))
            seen.append(kk)

    dr.ft_geqrf(A, nb, tol=NO_REFRESH, invariant_hook=hook)
    assert seen == [0]


def test_qr_pd_second_reflector_magnitude_closed_form():
    """Alg. 1's in-panel magnitude update (mck += |tau| m_v |y|) on a
    hand-solvable panel [x, c*v0, 0, ...]: the first reflector maps column 1
    to -c*v0, so before step j=1 its tile magnitudes are
    |c| e^T|v0_I| + (2/v0^T v0) e^T|v0_I| |c| v0^T v0 = 3|c| e^T|v0_I|, and
    the second reflector (of x' = -c*v0[1:], beta1 = -sign(x'_1)||x'||) gets
    m_v1(I) = (3|c| e^T|v0_I| + |beta1|*[row 1 in tile I]) / (|x'_1| + |beta1|)."""
    n, nb, c = 256, 32, -0.75
    nt = n // nb
    g = si.rng(43)
    x = g.uniform(-1.0, 1.0, size=n)
    h, _ = np.linalg.qr(x[:, None], mode="raw")
    v0 = np.r_[1.0, h[0, 1:]]
    A = np.zeros((n, n))
    A[:, 0] = x
    A[:, 1] = c * v0
    st = ck.State.alloc(A, nb)
    ck.encode(st, ck.Tiles(0, nt, 0, nt), ck.BOTH)
    up.qr_pd_alg1(st, 0)
    x1 = abs(c * v0[1])
    beta1 = abs(c) * np.linalg.norm(v0[1:])
    for I in range(nt):
        ev = np.abs(v0[I * nb:(I + 1) * nb]).sum()
        want = (3.0 * abs(c) * ev + (beta1 if I == 0 else 0.0)) / (x1 + beta1)
        _close(st.colmag[I, 1], want, ("m_v1", I))


def test_qr_tmu_magnitudes_closed_form_reflection():
    """A hand-solvable QR step: panel 0 = [x, 0, ..., 0] (one nontrivial
    reflector v, tau = 2/v^T v, all other tau = 0) and A2 = v g^T, which the
    reflector maps to H A2 = -v g^T.  The TMU rules give
    m_c(A2) = e^T|A2| + m_c(V)|W| with W = T^T V^T A2 = 2 e_0 g^T, i.e.
    e^T|v||g|^T + 2 e^T|v||g|^T = 3 e^T|H A2| per tile column, and likewise
    m_r(A2) = |A2|e + |V||T|^T|V|^T|A2|e = 3 |H A2| e per tile row.
    v comes from LAPACK (numpy.linalg.qr raw) of x."""
    n, nb = 256, 32
    nt = n // nb
    g = si.rng(41)
    x = g.uniform(-1.0, 1.0, size=n)
    h, _ = np.linalg.qr(x[:, None], mode="raw")
    v = np.r_[1.0, h[0, 1:]]  # LAPACK's unit-leading reflector of x
    gv = g.uniform(-1.0, 1.0, size=n - nb)
    A = np.zeros((n, n))
    A[:, 0] = x
    A[:, nb:] = np.outer(v, gv)
    st = ck.State.alloc(A, nb)
    ck.encode(st, ck.Tiles(0, nt, 0, nt), ck.BOTH)
    tau = up.qr_pd_alg1(st, 0)
    assert tau[0] == pytest.approx(2.0 / (v @ v), rel=1e-13) and np.all(tau[1:] == 0.0)
    V = up.qr_V(st, 0)
    T = up.qr_T(V, tau)
    Wm = up.qr_tmu_data(st, 0, V, T)
    up.qr_tmu_chk(st, 0, V, T, Wm)
    HA2 = -np.outer(v, gv)
    _close(st.A[:, nb:], HA2, "H A2")
    for I in range(nt):
        for J in range(1, nt):
            rs, cs = slice(I * nb, (I + 1) * nb), slice(J * nb, (J + 1) * nb)
            X = HA2[rs, (J - 1) * nb:J * nb]  # HA2 starts at column nb
            _close(st.colmag[I, cs], 3.0 * _colsum(X), ("col", I, J))
            _close(st.rowmag[rs, J], 3.0 * _rowsum(X), ("row", I, J))


def test_qr_magnitude_lower_bound_every_phase():
    n, nb = 256, 32
    A = si.general(n, seed=13)
    nt = n // nb

    def hook(st, k, phase):
        if phase == "pd":
            tv = [(I, k, ck.UNIT_LOWER if I == k else ck.GENERAL) for I in range(k, nt)]
            _lower_bounds(st, tv, ck.COL)
            _lower_bounds(st, [(k, k, ck.UPPER)], ck.ROW)
        else:
            _lower_bounds(st, [(k, J, ck.GENERAL) for J in range(k + 1, nt)], ck.ROW)
            _lower_bounds(st, [(I, J, ck.GENERAL) for I, J in ck.Tiles(k + 1, nt, k + 1, nt)], ck.BOTH)

    for tol in (NO_REFRESH, ck.Tol(refresh=True)):
        dr.ft_geqrf(A, nb, tol=tol, invariant_hook=hook)


# ---------------------------------------------------------------- refresh --
def test_refresh_rebases_clean_entries_only():
    """verify(refresh): every unflagged checksum entry takes the recomputed
    value and its magnitude the fresh e^T|X| (|X|e for rows); flagged
    entries keep their maintained values for locate/correct."""
    n, nb = 128, 32
    st = ck.State.alloc(si.general(n, seed=31), nb)
    nt = n // nb
    ck.encode(st, ck.Tiles(0, nt, 0, nt), ck.BOTH)
    exact = st.copy()
    st.colmag *= 7.0  # stale, inflated magnitudes
    st.rowmag *= 7.0
    st.colchk += 1e-15 * np.abs(st.colchk)  # tiny, unflagged drift
    st.A[37, 70] += 0.5  # one data error: flags column 70 and row 37
    exact.A[37, 70] = st.A[37, 70]
    ck.verify(st, ck.Tiles(0, nt, 0, nt), ck.BOTH, ck.Tol(refresh=True))
    ck.encode(exact, ck.Tiles(0, nt, 0, nt), ck.BOTH)  # checksums of the current data
    keep_c = np.zeros(st.colchk.shape[1], bool)
    keep_c[70] = True
    keep_r = np.zeros(st.rowchk.shape[0], bool)
    keep_r[37] = True
    assert np.array_equal(st.colchk[:, ~keep_c], exact.colchk[:, ~keep_c])
    assert np.array_equal(st.colmag[:, ~keep_c], exact.colmag[:, ~keep_c])
    assert np.array_equal(st.rowchk[~keep_r], exact.rowchk[~keep_r])
    assert np.array_equal(st.rowmag[~keep_r], exact.rowmag[~keep_r])
    assert st.colmag[1, 70] != exact.colmag[1, 70]  # flagged: untouched
    assert st.rowmag[37, 2] != exact.rowmag[37, 2]


def test_refresh_keeps_lu_thresholds_sharp():
    """DESIGN's refresh claim (c-6): without refresh, LU magnitudes compound
    the |U_kk^-1| / |L_kk^-1| factors from iteration to iteration until tau
    hides errors of every practical size; with refresh a mid-size error
    (a flip of mantissa bit 44: |delta| ~ 2^-8 |x|) is detected, located and
    fixed.  n=256 nb=32 U(-1,1)."""
    n, nb = 256, 32
    A = si.general(n, seed=5)
    lu, p = sla.lu_factor(A)
    ratios = {}

    for refresh in (False, True):
        worst = [0.0]

        def hook(st, k, phase):
            if phase != "tmu":
                return
            for I, J in ck.Tiles(k + 1, st.nt, k + 1, st.nt):
                X = ck.tile_view(st.A, I, J, nb, ck.GENERAL)
                worst[0] = max(worst[0], float((st.colmag[I, J * nb:(J + 1) * nb] / _colsum(X)).max()))

        dr.ft_getrf(A, nb, tol=ck.Tol(refresh=refresh), invariant_hook=hook)
        ratios[refresh] = worst[0]
    # gamma_32 ~ 3.6e-15: a ratio beyond 1e10 makes tau_e ~ 7e-5 * e^T|X|
    assert ratios[False] > 1e10 and ratios[True] < 1e3, ratios

    # a computation error in the trailing matrix after the 5th TMU
    inj = [dr.Inject(5, dr.AT_POST_TMU, dr.KIND_PERSIST, 0, 230, 235, (44,))]
    LU1, piv1, s1 = dr.ft_getrf(A, nb, tol=ck.Tol(refresh=True), inject=inj)
    assert s1.counts[0] >= 1 and s1.uncorrectable == 0
    assert np.abs(LU1 - lu).max() <= 1e-12 * np.abs(lu).max()
    LU0, piv0, s0 = dr.ft_getrf(A, nb, tol=ck.Tol(refresh=False), inject=inj)
    assert s0.counts[0] == 0  # undetected: the compounded tau swallowed it
    assert np.abs(LU0 - lu).max() > 1e-6 * np.abs(lu).max()
