"""ORACLE (test infrastructure only) — checksum maintenance through the
decomposition steps (§8 rows a4–a6), written step by step from the paper:

* checksums are updated "as if the checksums are an extended part of the
  original input matrix ... applying the same operation" (L149, §IV);
* full-checksum Cholesky: "transposing the column checksum of column panel to
  get row checksum" keeps full checksums through the TMU (L189, Table II);
* the a-priori round-off bound gamma_n·||A||·||B|| for C <- C − A·B
  (L124–L131) is carried per component as magnitude checksums (reading c-6).

Every function mutates a `checksum.State` in place and uses plain numpy /
scipy (triangular solves, matmuls) in float64.  Readings: c-6, c-12, c-13,
c-25.
"""
from __future__ import annotations

import numpy as np
import scipy.linalg as sla

from .checksum import State


def tri_inv(T, lower=True, unit=False):
    """Explicit T^-1 (used only for the magnitude rule of c-6)."""
    n = T.shape[0]
    return sla.solve_triangular(T, np.eye(n), lower=lower, unit_diagonal=unit, check_finite=False)


def potrf_lower(S):
    """LAPACK dpotrf('L') of a symmetric tile: (L, info) with info the
    1-based failing minor (0 on success)."""
    c, info = sla.lapack.dpotrf(S, lower=1, clean=1)
    return np.tril(c), int(info)


def chol_pd_rule(st: State, k: int):
    """c-12 PD: L_kk = chol(A_kk) (lower triangle of the tile, the LAPACK
    potrf 'L' convention), then c(L_kk) = c_sym(A_kk)·L_kk^{-T} and
    m_c(L_kk) = m_c(A_kk)·|L_kk^{-T}|.  Returns LAPACK-style info (0 or the
    1-based failing minor)."""
    nb = st.nb
    s = slice(k * nb, (k + 1) * nb)
    Akk = st.A[s, s]
    S = np.tril(Akk) + np.tril(Akk, -1).T
    L, info = potrf_lower(S)
    if info:
        return info
    st.A[s, s] = np.tril(L) + np.triu(Akk, 1)  # upper part of the tile untouched (potrf 'L')
    # c(L) L^T = c(A)  =>  c(L) = c(A) L^{-T}  (solve L · c(L)^T = c(A)^T)
    C = st.colchk[2 * k:2 * k + 2, s]
    st.colchk[2 * k:2 * k + 2, s] = sla.solve_triangular(L, C.T, lower=True, check_finite=False).T
    if st.colmag is not None:
        st.colmag[k, s] = st.colmag[k, s] @ np.abs(tri_inv(L).T)
    return 0


def chol_pu_data(st: State, k: int):
    """c-12 PU data step: L_ik = A_ik·L_kk^{-T} for the column panel."""
    nb, n = st.nb, st.A.shape[0]
    s = slice(k * nb, (k + 1) * nb)
    r1 = (k + 1) * nb
    L = np.tril(st.A[s, s])
    P = st.A[r1:n, s]
    st.A[r1:n, s] = sla.solve_triangular(L, P.T, lower=True, check_finite=False).T


def chol_pu_chk(st: State, k: int):
    """c-12 PU checksum step: c(L_ik) = c(A_ik)·L_kk^{-T}, m_c ← m_c·|L_kk^{-T}|."""
    nb = st.nb
    s = slice(k * nb, (k + 1) * nb)
    L = np.tril(st.A[s, s])
    C = st.colchk[2 * (k + 1):, s]
    st.colchk[2 * (k + 1):, s] = sla.solve_triangular(L, C.T, lower=True, check_finite=False).T
    if st.colmag is not None:
        st.colmag[k + 1:, s] = st.colmag[k + 1:, s] @ np.abs(tri_inv(L).T)


def chol_tmu_data(st: State, k: int, c0: int = None, c1: int = None):
    """c-12 TMU data step, every trailing tile (i ≥ j > k):
    A_ij −= L_ik L_jk^T on the lower triangle only (as DSYRK).  With a
    column range [c0, c1) (look-ahead, reading c-35) only those columns of
    the trailing matrix are updated."""
    nb, n = st.nb, st.A.shape[0]
    s = slice(k * nb, (k + 1) * nb)
    r1 = (k + 1) * nb
    c0 = r1 if c0 is None else c0
    c1 = n if c1 is None else c1
    L21 = st.A[r1:n, s].copy()
    upd = L21 @ L21[c0 - r1:c1 - r1].T  # rows r1:n, columns c0:c1
    rows = np.arange(r1, n)[:, None]
    cols = np.arange(c0, c1)[None, :]
    tri = rows >= cols
    st.A[r1:n, c0:c1][tri] -= upd[tri]


def chol_tmu_chk(st: State, k: int, c0: int = None, c1: int = None):
    """c-12 TMU checksum step: c(A_ij) −= c(L_ik)·L_jk^T,
    r(A_ij) −= L_ik·c(L_jk)^T (L189), m_c(A_ij) += m_c(L_ik)·|L_jk|^T,
    m_r(A_ij) += |L_ik|·m_c(L_jk)^T (c-6).  With a column range [c0, c1)
    (tile-aligned; look-ahead, reading c-35) only the tile columns j in it."""
    nb, n = st.nb, st.A.shape[0]
    s = slice(k * nb, (k + 1) * nb)
    r1 = (k + 1) * nb
    c0 = r1 if c0 is None else c0
    c1 = n if c1 is None else c1
    J0, J1 = c0 // nb, c1 // nb
    L21 = st.A[r1:n, s].copy()
    Lj = L21[c0 - r1:c1 - r1]
    cL = st.colchk[2 * (k + 1):, s].copy()
    cLj = cL[2 * (J0 - k - 1):2 * (J1 - k - 1)]
    st.colchk[2 * (k + 1):, c0:c1] -= cL @ Lj.T
    st.rowchk[r1:n, 2 * J0:2 * J1] -= L21 @ cLj.T
    if st.colmag is not None:
        mL = st.colmag[k + 1:, s].copy()
        mLj = mL[J0 - k - 1:J1 - k - 1]
        st.colmag[k + 1:, c0:c1] += mL @ np.abs(Lj).T
        st.rowmag[r1:n, J0:J1] += np.abs(L21) @ mLj.T


def chol_fig4a_repair(st: State, k: int, gi: int, gj: int, before: float, after: float, c0: int = 0,
                      c1: int = None):
    """Reading c-25 of Fig. 4a / L359 ('we can just fix the corresponding
    rows/columns in trailing matrix'): the panel re-check after the TMU fixed
    L[p, q] by E = after − before, but the TMU had used the bad value.  With
    ℓ = L_true[:, q]:  A_true = A_bad − E(e_p ℓ^T + ℓ e_p^T) + E² e_p e_p^T
    (lower part), c(A_I,i)[:, p'] −= E·c(L_I)[:, q'] for I ≥ i,
    r(A_i,J)[p', :] −= E·c(L_J)[:, q']^T for k < J ≤ i; magnitudes grow by
    |E| times the panel magnitude.  Guard: skipped when E is non-finite or
    |E| > 2^10·max|L_panel[:, q]|.  Returns 'applied', 'skipped' or None (not
    a panel element of iteration k).  A column range [c0, c1) (look-ahead,
    reading c-35) restricts the repair to the trailing columns that consumed
    the bad value: the tile column k+1 for the re-check after its update, the
    rest for the re-check after the rest of the TMU."""
    nb, n = st.nb, st.A.shape[0]
    c1 = n if c1 is None else c1
    r1 = (k + 1) * nb
    p, q = gi, gj
    if not (k * nb <= q < (k + 1) * nb and p >= r1):
        return None
    E = after - before
    mx = float(np.max(np.abs(st.A[r1:n, q])))
    if not (np.isfinite(E) and abs(E) <= 1024.0 * mx):
        return "skipped"
    i, pl, ql = p // nb, p % nb, q - k * nb
    ell = st.A[:, q]
    b0, b1 = max(r1, c0), min(p, c1)
    if b1 > b0:
        st.A[p, b0:b1] -= E * ell[b0:b1]
    if c0 <= p < c1:
        st.A[p + 1:n, p] -= E * ell[p + 1:n]
        st.A[p, p] -= 2.0 * E * ell[p] - E * E
    nt = n // nb
    if c0 <= p < c1:
        for I in range(i, nt):
            st.colchk[2 * I:2 * I + 2, i * nb + pl] -= E * st.colchk[2 * I:2 * I + 2, k * nb + ql]
            if st.colmag is not None:
                st.colmag[I, i * nb + pl] += abs(E) * st.colmag[I, k * nb + ql]
    for J in range(k + 1, i + 1):
        if not c0 <= J * nb < c1:
            continue
        st.rowchk[p, 2 * J:2 * J + 2] -= E * st.colchk[2 * J:2 * J + 2, k * nb + ql]
        if st.rowmag is not None:
            st.rowmag[p, J] += abs(E) * st.colmag[J, k * nb + ql]
    return "applied"


# ------------------------------------------------------------------- LU ----
def lu_swap_rule(st: State, p: int, q: int, cols, vals_p, vals_q, row_chk_cols=()):
    """Reading c-14 of the silent swap rule: exchanging global rows p and q
    (p' = p mod nb in tile P, q' in tile Q) changes the column checksums of
    every column `cols` by the moved values (x_p, x_q the values before the
    swap):  P != Q: c(P) += [1, p'+1]^T (x_q − x_p), c(Q) += [1, q'+1]^T (x_p − x_q);
    P == Q: c_w += (p' − q')(x_q − x_p); magnitudes follow |x|.  Row
    checksums (and row magnitudes) of the tile columns `row_chk_cols` move
    with the rows."""
    nb = st.nb
    P, Q, pl, ql = p // nb, q // nb, p % nb, q % nb
    d = np.asarray(vals_q, dtype=np.float64) - np.asarray(vals_p, dtype=np.float64)
    da = np.abs(vals_q) - np.abs(vals_p)
    if P != Q:
        st.colchk[2 * P, cols] += d
        st.colchk[2 * P + 1, cols] += (pl + 1) * d
        st.colchk[2 * Q, cols] -= d
        st.colchk[2 * Q + 1, cols] -= (ql + 1) * d
        if st.colmag is not None:
            st.colmag[P, cols] += da
            st.colmag[Q, cols] -= da
    else:
        st.colchk[2 * P + 1, cols] += (pl - ql) * d
    for J in row_chk_cols:
        st.rowchk[[p, q], 2 * J:2 * J + 2] = st.rowchk[[q, p], 2 * J:2 * J + 2]
        if st.rowmag is not None:
            st.rowmag[[p, q], J] = st.rowmag[[q, p], J]


def lu_panel_getrf(st: State, k: int):
    """c-13 PD, factor step: LAPACK dgetrf of the column panel
    P = A[k·nb:, k·nb:(k+1)·nb] (partial pivoting, idamax ties → first).
    Does not touch the state.  Returns (lu_panel, ipiv 0-based global,
    info, pre-PD panel copy)."""
    nb, n = st.nb, st.A.shape[0]
    r0, r1 = k * nb, (k + 1) * nb
    P0 = st.A[r0:n, r0:r1].copy()
    lu, piv, info = sla.lapack.dgetrf(P0.copy())
    return lu, r0 + np.asarray(piv, dtype=np.int64), int(info), P0


def lu_swap_rows(ipiv, k, nb):
    """The rows a panel's pivot sequence moves (each swap p = k·nb + j <-> ipiv[j])."""
    rows = []
    for j, q in enumerate(ipiv):
        p = k * nb + j
        if p != int(q):
            rows += [p, int(q)]
    return sorted(set(rows))


def lu_pd_apply(st: State, k: int, lu, ipiv, P0, part: str = "all"):
    """c-13/c-14 PD, apply step: the row swaps on the left (factored L
    panels, c only) and right (trailing, c and r) columns with the swap rule,
    the panel's own column checksums swapped with the PRE-PD copy (L430),
    then c(L_I) = c(P~_I)·U_kk^{-1} (L_kk in UNIT_LOWER view) and
    r(U_kk) = L_kk^{-1}·r(P~_kk), magnitudes by |U_kk^{-1}|, |L_kk^{-1}| (c-6).
    part (look-ahead, reading c-35): "panel" = everything inside the column
    panel (its columns' deltas, the row checksums of tile column k, the
    factor, the rules); "outside" = the swaps of every other column with
    their deltas and the row checksums of tile columns > k.  The two touch
    disjoint entries, so "panel" then "outside" equals "all"."""
    nb, n = st.nb, st.A.shape[0]
    nt = n // nb
    r0, r1 = k * nb, (k + 1) * nb
    copy = P0.copy() if P0 is not None else None
    panel_cols = np.arange(r0, r1)
    left_cols = np.arange(0, r0)
    right_cols = np.arange(r1, n)
    inside, outside = part in ("all", "panel"), part in ("all", "outside")
    for j in range(nb):
        p, q = r0 + j, int(ipiv[j])
        if p == q:
            continue
        if inside:
            lu_swap_rule(st, p, q, panel_cols, copy[p - r0].copy(), copy[q - r0].copy(),
                         row_chk_cols=range(k, nt) if part == "all" else range(k, k + 1))
            copy[[p - r0, q - r0]] = copy[[q - r0, p - r0]]
        if not outside:
            continue
        if part == "outside":
            lu_swap_rule(st, p, q, [], (), (), row_chk_cols=range(k + 1, nt))
        if r0 > 0:
            lu_swap_rule(st, p, q, left_cols, st.A[p, :r0].copy(), st.A[q, :r0].copy())
        if r1 < n:
            lu_swap_rule(st, p, q, right_cols, st.A[p, r1:].copy(), st.A[q, r1:].copy())
        st.A[[p, q], :r0] = st.A[[q, p], :r0]
        st.A[[p, q], r1:] = st.A[[q, p], r1:]
    if not inside:
        return
    st.A[r0:n, r0:r1] = lu
    U = np.triu(lu[:nb, :nb])
    Lkk = np.tril(lu[:nb, :nb], -1) + np.eye(nb)
    Uinv = tri_inv(U, lower=False)
    Linv = tri_inv(Lkk, lower=True, unit=True)
    cs = slice(r0, r1)
    st.colchk[2 * k:, cs] = st.colchk[2 * k:, cs] @ Uinv
    st.rowchk[r0:r1, 2 * k:2 * k + 2] = Linv @ st.rowchk[r0:r1, 2 * k:2 * k + 2]
    if st.colmag is not None:
        st.colmag[k:, cs] = st.colmag[k:, cs] @ np.abs(Uinv)
        st.rowmag[r0:r1, k] = np.abs(Linv) @ st.rowmag[r0:r1, k]


def lu_pd_undo(st: State, k: int, ipiv):
    """f1 (L430) for LU: take back the row swaps a PD applied outside its
    panel — the same transpositions in reverse order (a transposition is its
    own inverse), with the c-14 swap rule on the left and right columns and
    the row checksums of tile columns > k moving back with their rows.  The
    panel itself and its checksums are restored from the pre-PD copy by the
    caller."""
    nb, n = st.nb, st.A.shape[0]
    nt = n // nb
    r0, r1 = k * nb, (k + 1) * nb
    left_cols = np.arange(0, r0)
    right_cols = np.arange(r1, n)
    for j in reversed(range(nb)):
        p, q = r0 + j, int(ipiv[j])
        if p == q:
            continue
        if r0 > 0:
            lu_swap_rule(st, p, q, left_cols, st.A[p, :r0].copy(), st.A[q, :r0].copy())
        if r1 < n:
            lu_swap_rule(st, p, q, right_cols, st.A[p, r1:].copy(), st.A[q, r1:].copy(),
                         row_chk_cols=range(k + 1, nt))
        st.A[[p, q], :r0] = st.A[[q, p], :r0]
        st.A[[p, q], r1:] = st.A[[q, p], r1:]


def lu_pd(st: State, k: int):
    """Factor + apply (no pre-swap check): returns (ipiv_global, info)."""
    lu, ipiv, info, P0 = lu_panel_getrf(st, k)
    lu_pd_apply(st, k, lu, ipiv, P0)
    return ipiv, info


def lu_pu_data(st: State, k: int):
    """c-13 PU data step: U_kJ = L_kk^{-1}·A_kJ for the row panel."""
    nb, n = st.nb, st.A.shape[0]
    r0, r1 = k * nb, (k + 1) * nb
    Lkk = np.tril(st.A[r0:r1, r0:r1], -1) + np.eye(nb)
    st.A[r0:r1, r1:n] = sla.solve_triangular(Lkk, st.A[r0:r1, r1:n], lower=True, unit_diagonal=True,
                                             check_finite=False)


def lu_pu_chk(st: State, k: int):
    """c-13 PU checksum step: r(U_kJ) = L_kk^{-1}·r(A_kJ), m_r ← |L_kk^{-1}|·m_r."""
    nb = st.nb
    r0, r1 = k * nb, (k + 1) * nb
    Lkk = np.tril(st.A[r0:r1, r0:r1], -1) + np.eye(nb)
    st.rowchk[r0:r1, 2 * (k + 1):] = sla.solve_triangular(Lkk, st.rowchk[r0:r1, 2 * (k + 1):], lower=True,
                                                          unit_diagonal=True, check_finite=False)
    if st.rowmag is not None:
        st.rowmag[r0:r1, k + 1:] = np.abs(tri_inv(Lkk, lower=True, unit=True)) @ st.rowmag[r0:r1, k + 1:]


def lu_tmu_data(st: State, k: int, c0: int = None, c1: int = None):
    """c-13 TMU data step: A_IJ −= L_Ik·U_kJ for every trailing tile (tile
    columns in [c0, c1) only, for the look-ahead split, reading c-35)."""
    nb, n = st.nb, st.A.shape[0]
    r0, r1 = k * nb, (k + 1) * nb
    c0 = r1 if c0 is None else c0
    c1 = n if c1 is None else c1
    st.A[r1:n, c0:c1] -= st.A[r1:n, r0:r1] @ st.A[r0:r1, c0:c1]


def lu_tmu_chk(st: State, k: int, c0: int = None, c1: int = None):
    """c-13 TMU checksum step: c(A_IJ) −= c(L_Ik)·U_kJ, r(A_IJ) −= L_Ik·r(U_kJ);
    m_c += m_c(L)·|U|, m_r += |L|·m_r(U) (c-6).  Tile-aligned column range
    [c0, c1) as in lu_tmu_data."""
    nb, n = st.nb, st.A.shape[0]
    r0, r1 = k * nb, (k + 1) * nb
    c0 = r1 if c0 is None else c0
    c1 = n if c1 is None else c1
    J0, J1 = c0 // nb, c1 // nb
    L21, U1j = st.A[r1:n, r0:r1], st.A[r0:r1, c0:c1]
    st.colchk[2 * (k + 1):, c0:c1] -= st.colchk[2 * (k + 1):, r0:r1] @ U1j
    st.rowchk[r1:n, 2 * J0:2 * J1] -= L21 @ st.rowchk[r0:r1, 2 * J0:2 * J1]
    if st.colmag is not None:
        st.colmag[k + 1:, c0:c1] += st.colmag[k + 1:, r0:r1] @ np.abs(U1j)
        st.rowmag[r1:n, J0:J1] += np.abs(L21) @ st.rowmag[r0:r1, J0:J1]


def lu_fig4a_repair(st: State, k: int, gi: int, gj: int, before: float, after: float, c0: int = 0,
                    c1: int = None):
    """Reading c-25 for LU: the post-TMU re-check corrected a panel element by
    E = after − before; the TMU had consumed the bad value.
    L21[p, q] (column panel): A[p, r1:] −= E·U[q, r1:], r(A_i,J)[p', :] −= E·r(U_J)[q, :]
      (c(A) was built from the good c(L), so only data and r change); m_r += |E|·m_r(U).
    U12[q, c] (row panel): A[r1:, c] −= L21[:, q]·E, c(A_I,j)[:, c'] −= c(L_I)[:, q]·E
      (r(A) was built from the good r(U)); m_c += |E|·m_c(L).
    Guard as in Cholesky (2^10 × max |panel line|, finite).  A column range
    [c0, c1) (look-ahead, reading c-35) restricts the repair to the trailing
    columns whose update consumed the bad value."""
    nb, n = st.nb, st.A.shape[0]
    nt = n // nb
    c1 = n if c1 is None else c1
    r0, r1 = k * nb, (k + 1) * nb
    E = after - before
    if r0 <= gj < r1 and gi >= r1:  # element of L21
        p, q = gi, gj - r0
        mx = float(np.max(np.abs(st.A[r1:n, gj])))
        if not (np.isfinite(E) and abs(E) <= 1024.0 * mx):
            return "skipped"
        b0, b1 = max(r1, c0), min(n, c1)
        st.A[p, b0:b1] -= E * st.A[r0 + q, b0:b1]
        for J in range(k + 1, nt):
            if not c0 <= J * nb < c1:
                continue
            st.rowchk[p, 2 * J:2 * J + 2] -= E * st.rowchk[r0 + q, 2 * J:2 * J + 2]
            if st.rowmag is not None:
                st.rowmag[p, J] += abs(E) * st.rowmag[r0 + q, J]
        return "applied"
    if r0 <= gi < r1 and gj >= r1:  # element of U12
        q, c = gi - r0, gj
        mx = float(np.max(np.abs(st.A[gi, r1:n])))
        if not (np.isfinite(E) and abs(E) <= 1024.0 * mx):
            return "skipped"
        if not c0 <= c < c1:
            return "applied"
        st.A[r1:n, c] -= st.A[r1:n, r0 + q] * E
        for I in range(k + 1, nt):
            st.colchk[2 * I:2 * I + 2, c] -= E * st.colchk[2 * I:2 * I + 2, r0 + q]
            if st.colmag is not None:
                st.colmag[I, c] += abs(E) * st.colmag[I, r0 + q]
        return "applied"
    return None


# ------------------------------------------------------------------- QR ----
def _panel_weights(nb, nt_rows):
    """W (2·nt_rows × nt_rows·nb): rows 2I / 2I+1 hold v1 / v2 of tile row I
    of the panel (tile-local, 1-based; L108)."""
    W = np.zeros((2 * nt_rows, nt_rows * nb))
    v1, v2 = np.ones(nb), np.arange(1, nb + 1, dtype=np.float64)
    for I in range(nt_rows):
        W[2 * I, I * nb:(I + 1) * nb] = v1
        W[2 * I + 1, I * nb:(I + 1) * nb] = v2
    return W


def qr_pd_alg1(st: State, k: int):
    """Algorithm 1 (L228–L235, reconstruction c-15) with LAPACK's dlarfg
    conventions (v(1) = 1, tau, beta = −sign(x1)·||x||; tau = 0 when x(2:) = 0):
    Householder QR of the column panel P = A[k·nb:, k·nb:(k+1)·nb] extended
    by its column checksums ck (per tile [v1 v2]^T P, the 'checksum row') and
    its row checksums rck (P [v1 v2], the 'checksum column').  For j = 0..nb−1:
      x = P[j:, j];  c_x = ck[:, j] − W[:, :j] P[:j, j]   (checksum of x from
                                       the trusted checksum minus finished rows)
      beta, tau, v = dlarfg(x);  v_ck = (c_x − beta·W[:, j]) / (x1 − beta)
      y = v^T P[j:, j+1:];  P[j:, j+1:] −= tau v y;  ck[:, j+1:] −= tau v_ck y
      rck[j:] −= tau v (v^T rck[j:])
      store beta, v(2:) in P[:, j] and v_ck in ck[:, j]  (= c(V) in UNIT_LOWER view)
    Magnitudes (c-6): m_x = mck[:, j]; m_v = (m_x + |beta|·[row j in tile]) / |x1 − beta|;
    mck[:, j+1:] += |tau| m_v |y|;  after the loop m_r += |V| (|T|^T (|V|^T m_r)).
    At the end rck = Q^T P [v1 v2] = [r(R); 0].  Returns tau (nb)."""
    nb, n = st.nb, st.A.shape[0]
    nt = n // nb
    r0, r1 = k * nb, (k + 1) * nb
    m = n - r0
    P = st.A[r0:n, r0:r1].copy()
    W = _panel_weights(nb, nt - k)
    ck = st.colchk[2 * k:, r0:r1].copy()
    rck = st.rowchk[r0:n, 2 * k:2 * k + 2].copy()
    mags = st.colmag is not None
    if mags:
        mck = st.colmag[k:, r0:r1].copy()
        mr = st.rowmag[r0:n, k].copy()
    tau = np.zeros(nb)
    for j in range(nb):
        x = P[j:, j].copy()
        c_x = ck[:, j] - W[:, :j] @ P[:j, j]
        alpha = x[0]
        xnorm = float(np.linalg.norm(x[1:]))
        e_row = (W[:, j] != 0).astype(np.float64)[0::2]  # tiles holding row j
        if xnorm == 0.0:
            t, beta = 0.0, alpha
            v = np.zeros_like(x)
            v[0] = 1.0
            v_ck = W[:, j].copy()
            if mags:
                m_v = e_row.copy()
        else:
            beta = -np.copysign(np.hypot(alpha, xnorm), alpha)
            t = (beta - alpha) / beta
            v = x / (alpha - beta)
            v[0] = 1.0
            v_ck = (c_x - beta * W[:, j]) / (alpha - beta)
            if mags:
                m_v = (mck[:, j] + abs(beta) * e_row) / abs(alpha - beta)
        tau[j] = t
        if j + 1 < nb:
            y = v @ P[j:, j + 1:]
            P[j:, j + 1:] -= t * np.outer(v, y)
            ck[:, j + 1:] -= t * np.outer(v_ck, y)
            if mags:
                mck[:, j + 1:] += abs(t) * np.outer(m_v, np.abs(y))
        yr = v @ rck[j:]
        rck[j:] -= t * np.outer(v, yr)
        P[j, j] = beta
        P[j + 1:, j] = v[1:]
        ck[:, j] = v_ck
        if mags:
            mck[:, j] = m_v
    st.A[r0:n, r0:r1] = P
    st.colchk[2 * k:, r0:r1] = ck
    st.rowchk[r0:n, 2 * k:2 * k + 2] = rck
    if mags:
        st.colmag[k:, r0:r1] = mck
        # rck = Q^T r(P), Q^T = I − V T^T V^T: m_r += |V| (|T|^T (|V|^T m_r)) (c-6)
        V = np.tril(P, -1)
        V[:nb, :nb] += np.eye(nb)
        T = qr_T(V, tau)
        st.rowmag[r0:n, k] = qr_rowmag_rule(V, T, mr)
    return tau


def qr_rowmag_rule(V, T, mr):
    """Row magnitudes through r <- (I − V T^T V^T) r, the QR row rule of both
    the PD (r(R) = Q^T r(P)) and the TMU (c-6): m_r + |V| (|T|^T (|V|^T m_r))."""
    return mr + np.abs(V) @ (np.abs(T).T @ (np.abs(V).T @ mr))


def qr_V(st: State, k: int):
    """V (unit lower trapezoidal) of panel k as stored by dgeqrf."""
    nb, n = st.nb, st.A.shape[0]
    r0, r1 = k * nb, (k + 1) * nb
    V = np.tril(st.A[r0:n, r0:r1], -1)
    V[:nb, :nb] += np.eye(nb)
    return V


def qr_T(V, tau):
    """CTF (the paper's 'computing triangular factor', L238; LAPACK dlarft,
    forward, columnwise): T[j,j] = tau_j, T[:j, j] = −tau_j T[:j,:j] V[:, :j]^T v_j."""
    nb = V.shape[1]
    T = np.zeros((nb, nb))
    for j in range(nb):
        T[j, j] = tau[j]
        if j:
            T[:j, j] = -tau[j] * (T[:j, :j] @ (V[:, :j].T @ V[:, j]))
    return T


def qr_ctf_check(V, T, prec="f64", scale=1.0):
    """f2, the CTF check (L263: "Error in T can be detected by verifying the
    orthogonality of (I − V T V^T) ... recover the corrupted T by re-computing
    it using V").  Q = I − V T V^T is orthogonal iff V (T + T^T − T^T V^T V T) V^T
    = 0, i.e. for V of full column rank iff E = T^T (V^T V) T − T − T^T = 0.
    Reading c-29: flag iff some |E_ij| > scale·4·γ_{m+nb}·(a_i a_j + |T_ij| +
    |T_ji|) with a = |T|^T ‖v‖ (‖v_k‖ = column norms of V, so that
    |V|^T |V| ≤ ‖v‖ ‖v‖^T bounds the rounding of V^T V; the |T| terms cover
    2/τ_j vs v_j^T v_j); a non-finite E_ij or bound is flagged.  Returns
    (flagged entries, E)."""
    m, nb = V.shape
    S = V.T @ V
    E = T.T @ S @ T - T - T.T
    a = np.abs(T).T @ np.sqrt(np.diag(S))
    u = 2.0 ** -53 if prec == "f64" else 2.0 ** -24
    g = (m + nb) * u / (1.0 - (m + nb) * u)
    bound = scale * 4.0 * g * (np.outer(a, a) + np.abs(T) + np.abs(T).T)
    with np.errstate(invalid="ignore"):
        bad = ~np.isfinite(E) | ~np.isfinite(bound) | ~(np.abs(E) <= bound)
    return int(np.count_nonzero(bad)), E


def qr_tmu_data(st: State, k: int, V, T):
    """QR TMU data step (Table III): A2 ← (I − V T V^T)^T A2 = A2 − V (T^T V^T A2)
    for A2 = A[k·nb:, (k+1)·nb:] (its first nb rows become R12)."""
    nb, n = st.nb, st.A.shape[0]
    r0, r1 = k * nb, (k + 1) * nb
    A2 = st.A[r0:n, r1:n]
    Wm = T.T @ (V.T @ A2)
    st.A[r0:n, r1:n] = A2 - V @ Wm
    return Wm


def qr_tmu_chk(st: State, k: int, V, T, Wm):
    """QR TMU checksum step (Table III, red symbols; c-15): with W = T^T V^T A2,
    c(A2) −= c(V)·W and r(A2) −= V·(T^T V^T r(A2)); magnitudes
    m_c += m_c(V)|W|, m_r += |V| (|T|^T (|V|^T m_r)) (c-6)."""
    nb, n = st.nb, st.A.shape[0]
    r0, r1 = k * nb, (k + 1) * nb
    cV = st.colchk[2 * k:, r0:r1]
    st.colchk[2 * k:, r1:n] -= cV @ Wm
    rA = st.rowchk[r0:n, 2 * (k + 1):]
    st.rowchk[r0:n, 2 * (k + 1):] = rA - V @ (T.T @ (V.T @ rA))
    if st.colmag is not None:
        st.colmag[k:, r1:n] += st.colmag[k:, r0:r1] @ np.abs(Wm)
        st.rowmag[r0:n, k + 1:] = qr_rowmag_rule(V, T, st.rowmag[r0:n, k + 1:])
