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


def chol_tmu_data(st: State, k: int):
    """c-12 TMU data step, every trailing tile (i ≥ j > k):
    A_ij −= L_ik L_jk^T on the lower triangle only (as DSYRK)."""
    nb, n = st.nb, st.A.shape[0]
    s = slice(k * nb, (k + 1) * nb)
    r1 = (k + 1) * nb
    L21 = st.A[r1:n, s].copy()
    upd = L21 @ L21.T
    tri = np.tril(np.ones((n - r1, n - r1), dtype=bool))
    st.A[r1:n, r1:n][tri] -= upd[tri]


def chol_tmu_chk(st: State, k: int):
    """c-12 TMU checksum step: c(A_ij) −= c(L_ik)·L_jk^T,
    r(A_ij) −= L_ik·c(L_jk)^T (L189), m_c(A_ij) += m_c(L_ik)·|L_jk|^T,
    m_r(A_ij) += |L_ik|·m_c(L_jk)^T (c-6)."""
    nb, n = st.nb, st.A.shape[0]
    s = slice(k * nb, (k + 1) * nb)
    r1 = (k + 1) * nb
    L21 = st.A[r1:n, s].copy()
    cL = st.colchk[2 * (k + 1):, s].copy()
    st.colchk[2 * (k + 1):, r1:n] -= cL @ L21.T
    st.rowchk[r1:n, 2 * (k + 1):] -= L21 @ cL.T
    if st.colmag is not None:
        mL = st.colmag[k + 1:, s].copy()
        st.colmag[k + 1:, r1:n] += mL @ np.abs(L21).T
        st.rowmag[r1:n, k + 1:] += np.abs(L21) @ mL.T


def chol_fig4a_repair(st: State, k: int, gi: int, gj: int, before: float, after: float):
    """Reading c-25 of Fig. 4a / L359 ('we can just fix the corresponding
    rows/columns in trailing matrix'): the panel re-check after the TMU fixed
    L[p, q] by E = after − before, but the TMU had used the bad value.  With
    ℓ = L_true[:, q]:  A_true = A_bad − E(e_p ℓ^T + ℓ e_p^T) + E² e_p e_p^T
    (lower part), c(A_I,i)[:, p'] −= E·c(L_I)[:, q'] for I ≥ i,
    r(A_i,J)[p', :] −= E·c(L_J)[:, q']^T for k < J ≤ i; magnitudes grow by
    |E| times the panel magnitude.  Guard: skipped when E is non-finite or
    |E| > 2^10·max|L_panel[:, q]|.  Returns 'applied', 'skipped' or None (not
    a panel element of iteration k)."""
    nb, n = st.nb, st.A.shape[0]
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
    st.A[p, r1:p] -= E * ell[r1:p]
    st.A[p + 1:n, p] -= E * ell[p + 1:n]
    st.A[p, p] -= 2.0 * E * ell[p] - E * E
    nt = n // nb
    for I in range(i, nt):
        st.colchk[2 * I:2 * I + 2, i * nb + pl] -= E * st.colchk[2 * I:2 * I + 2, k * nb + ql]
        if st.colmag is not None:
            st.colmag[I, i * nb + pl] += abs(E) * st.colmag[I, k * nb + ql]
    for J in range(k + 1, i + 1):
        st.rowchk[p, 2 * J:2 * J + 2] -= E * st.colchk[2 * J:2 * J + 2, k * nb + ql]
        if st.rowmag is not None:
            st.rowmag[p, J] += abs(E) * st.colmag[J, k * nb + ql]
    return "applied"
