"""ORACLE (test infrastructure only) — per-tile weighted checksums: encode,
verify, locate, classify and correct.  Paper: PAPER.md §III.B (L108–L133),
§VII.D (L432–L434), §VIII.A (L444–L446); readings c-2 … c-11 of SURVEY §8c
(restated in DESIGN.md §4).

Everything is float64 numpy, one tile at a time, in the paper's notation:

  c(X) = [v1 v2]^T X      (2 x nb)   column checksum      (L111, L446)
  r(X) = X [v1 v2]        (nb x 2)   row checksum         (L111, L446)
  v1 = (1,…,1), v2 = (1,2,…,nb)  — tile-local, 1-based    (L108)
  delta = c(X) - recal_c(X)                                (L118–L120)
  detect |delta_1| > e_c; row = round(delta_2/delta_1)     (L122)

The matrix state is a `State`: the data A plus the maintained checksum arrays
(colchk (2·m/nb)×n, rowchk m×(2·n/nb)) and magnitude arrays
(colmag (m/nb)×n, rowmag m×(n/nb)) that carry the running e^T|X| used by the
threshold (reading c-6).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

# views (reading c-3) -------------------------------------------------------
GENERAL, LOWER, UNIT_LOWER, UPPER, SYM_LOWER = 0, 1, 2, 3, 4
# which checksums exist / are checked (reading c-9)
COL, ROW, BOTH = 1, 2, 3
# tolerance kinds (reading c-6)
TOL_MAGNITUDE, TOL_POSTERIORI = 0, 1
# classes (reading c-11)
CLS_CLEAN, CLS_0D, CLS_1D_ROW, CLS_1D_COL, CLS_SYM_CROSS = 0, 1, 2, 3, 4
CLS_CHK_CORRUPT, CLS_STALE_R, CLS_STALE_C, CLS_2D = 5, 6, 7, 8
# fix-record kinds
FIX_DATA, FIX_COLCHK, FIX_ROWCHK = 0, 1, 2
# per-tile status bits written by verify
ST_COL, ST_ROW, ST_NONFINITE, ST_UNCORRECTABLE = 1, 2, 4, 8


def unit_roundoff(prec: str) -> float:
    """u: 2^-53 for IEEE double (the paper's 'u ≈ 1e-16', L133), 2^-24 for
    single (fp32 is a BASELINE addition, reading c-21)."""
    return 2.0 ** -53 if prec == "f64" else 2.0 ** -24


def gamma(k: int, u: float) -> float:
    """gamma_k = k·u / (1 − k·u)  (L133)."""
    return k * u / (1.0 - k * u)


def weights(nb: int):
    """v1 = (1,…,1)^T, v2 = (1,2,…,nb)^T (L108; tile-local, 1-based: c-2)."""
    return np.ones(nb), np.arange(1, nb + 1, dtype=np.float64)


@dataclass
class State:
    """Matrix + maintained checksums (column-major semantics irrelevant here:
    A[i, j] is row i, column j)."""

    A: np.ndarray
    nb: int
    prec: str = "f64"
    colchk: np.ndarray = None
    rowchk: np.ndarray = None
    colmag: np.ndarray = None
    rowmag: np.ndarray = None

    @classmethod
    def alloc(cls, A, nb, prec="f64", mags=True):
        m, n = A.shape
        assert m % nb == 0 and n % nb == 0, "v1 requires m, n multiples of nb (reading c-22)"
        st = cls(A=np.array(A, dtype=np.float64), nb=nb, prec=prec)
        st.colchk = np.zeros((2 * m // nb, n))
        st.rowchk = np.zeros((m, 2 * n // nb))
        if mags:
            st.colmag = np.zeros((m // nb, n))
            st.rowmag = np.zeros((m, n // nb))
        return st

    @property
    def mt(self):
        return self.A.shape[0] // self.nb

    @property
    def nt(self):
        return self.A.shape[1] // self.nb

    def copy(self):
        c = lambda x: None if x is None else x.copy()
        return State(c(self.A), self.nb, self.prec, c(self.colchk), c(self.rowchk), c(self.colmag), c(self.rowmag))


@dataclass
class Tiles:
    """Half-open tile ranges; lower_only keeps I >= J (Cholesky); diag_view
    applies to tiles with I == J, all others are GENERAL."""

    I0: int
    I1: int
    J0: int
    J1: int
    lower_only: bool = False
    diag_view: int = GENERAL

    def __iter__(self):
        for J in range(self.J0, self.J1):
            for I in range(self.I0, self.I1):
                if self.lower_only and I < J:
                    continue
                yield I, J

    def view(self, I, J):
        return self.diag_view if I == J else GENERAL


@dataclass
class Tol:
    """Threshold policy (reading c-6): tau_e = scale·2·gamma_nb·m,
    tau_w = nb·tau_e, m = maintained magnitude (TOL_MAGNITUDE, when the state
    carries magnitude arrays) or e^T|X| of the current tile (fresh encode, or
    TOL_POSTERIORI)."""

    kind: int = TOL_MAGNITUDE
    scale: float = 1.0
    refresh: bool = False  # rebase clean entries on the recomputed checksums (c-6)


@dataclass
class Fix:
    gi: int
    gj: int
    before: float
    after: float
    cls: int
    kind: int = FIX_DATA


# ------------------------------------------------------------------ views --
def tile_view(A, I, J, nb, view):
    """The nb×nb block X the checksums describe (reading c-3):
    GENERAL — the stored block; LOWER — upper part read as 0; UNIT_LOWER —
    strictly-lower part plus an implicit unit diagonal; UPPER — lower part read
    as 0; SYM_LOWER — the symmetric block mirrored from the stored lower
    triangle, X[i, j] = A[max(i,j), min(i,j)]."""
    X = np.array(A[I * nb:(I + 1) * nb, J * nb:(J + 1) * nb], dtype=np.float64)
    if view == GENERAL:
        return X
    if view == LOWER:
        return np.tril(X)
    if view == UNIT_LOWER:
        return np.tril(X, -1) + np.eye(nb)
    if view == UPPER:
        return np.triu(X)
    if view == SYM_LOWER:
        L = np.tril(X)
        return L + np.tril(X, -1).T
    raise ValueError(view)


def live(view, i, j):
    """Whether view element (i, j) is backed by storage that can hold an error."""
    if view == LOWER:
        return i >= j
    if view == UNIT_LOWER:
        return i > j
    if view == UPPER:
        return i <= j
    return True


def stored_index(view, i, j):
    """Storage element behind view element (i, j) (SYM_LOWER mirrors, c-3)."""
    if view == SYM_LOWER:
        return max(i, j), min(i, j)
    return i, j


# ----------------------------------------------------------------- encode --
def encode_tile(X):
    """c = [v1 v2]^T X, r = X [v1 v2] (L111/L446) and the magnitude sums
    m_c = v1^T |X|, m_r = |X| v1 (reading c-6).  Pins: tests/test_oracle_checksum.py
    (closed forms, exact integer sums, fsum bound)."""
    nb = X.shape[0]
    v1, v2 = weights(nb)
    V = np.stack([v1, v2], axis=1)  # nb x 2
    c = V.T @ X  # 2 x nb
    r = X @ V  # nb x 2
    aX = np.abs(X)
    return c, r, v1 @ aX, aX @ v1


def _cols(st, J):
    return slice(J * st.nb, (J + 1) * st.nb)


def _rows(st, I):
    return slice(I * st.nb, (I + 1) * st.nb)


def encode(st: State, tiles: Tiles, which=BOTH):
    """abft_encode: write c / r (and magnitudes, when the state has them) of
    every selected tile (§8 row a1)."""
    for I, J in tiles:
        X = tile_view(st.A, I, J, st.nb, tiles.view(I, J))
        c, r, mc, mr = encode_tile(X)
        if which & COL:
            st.colchk[2 * I:2 * I + 2, _cols(st, J)] = c
            if st.colmag is not None:
                st.colmag[I, _cols(st, J)] = mc
        if which & ROW:
            st.rowchk[_rows(st, I), 2 * J:2 * J + 2] = r
            if st.rowmag is not None:
                st.rowmag[_rows(st, I), J] = mr


# ----------------------------------------------------------------- verify --
@dataclass
class TileCheck:
    I: int
    J: int
    view: int
    X: np.ndarray
    dc: np.ndarray = None  # 2 x nb: delta = maintained - recomputed (L119)
    dr: np.ndarray = None  # nb x 2
    tc: np.ndarray = None  # tau_e per column
    tr: np.ndarray = None  # tau_e per row
    fce: np.ndarray = None
    fcw: np.ndarray = None
    fre: np.ndarray = None
    frw: np.ndarray = None
    nonfinite: bool = False
    _use_mag: bool = False

    @property
    def Fc(self):
        return [] if self.fce is None else [int(j) for j in np.nonzero(self.fce | self.fcw)[0]]

    @property
    def Fr(self):
        return [] if self.fre is None else [int(i) for i in np.nonzero(self.fre | self.frw)[0]]

    @property
    def status(self):
        s = 0
        if self.Fc:
            s |= ST_COL
        if self.Fr:
            s |= ST_ROW
        if self.nonfinite:
            s |= ST_NONFINITE
        return s


def tau_e(st: State, m):
    """tau_e = scale·2·gamma_nb·m (reading c-6; the paper's a-priori bound
    gamma_n·||A||·||B|| of L126–L131 applied per checksum component)."""
    return 2.0 * gamma(st.nb, unit_roundoff(st.prec)) * m


def _flag(d, t):
    """|delta| > tau, or delta non-finite (reading c-7)."""
    with np.errstate(invalid="ignore"):
        return ~np.isfinite(d) | (np.abs(d) > t)


def check_tile(st: State, I, J, view, which, tol: Tol = Tol()):
    """Recompute (L116 'recal_c'), delta = maintained − recomputed (L119),
    flag columns/rows whose e- or w-residual exceeds tau (L122, c-6)."""
    nb = st.nb
    X = tile_view(st.A, I, J, nb, view)
    c, r, mc, mr = encode_tile(X)
    tc = TileCheck(I, J, view, X)
    use_mag = tol.kind == TOL_MAGNITUDE and st.colmag is not None
    with np.errstate(invalid="ignore", over="ignore"):
        if which & COL:
            tc.dc = st.colchk[2 * I:2 * I + 2, _cols(st, J)] - c
            m = st.colmag[I, _cols(st, J)] if use_mag else mc
            tc.tc = tol.scale * tau_e(st, m)
            tc.fce = _flag(tc.dc[0], tc.tc)
            tc.fcw = _flag(tc.dc[1], nb * tc.tc)
            tc.nonfinite |= bool(~np.all(np.isfinite(tc.dc)))
        if which & ROW:
            tc.dr = st.rowchk[_rows(st, I), 2 * J:2 * J + 2] - r
            m = st.rowmag[_rows(st, I), J] if use_mag else mr
            tc.tr = tol.scale * tau_e(st, m)
            tc.fre = _flag(tc.dr[:, 0], tc.tr)
            tc.frw = _flag(tc.dr[:, 1], nb * tc.tr)
            tc.nonfinite |= bool(~np.all(np.isfinite(tc.dr)))
    return tc


def verify(st: State, tiles: Tiles, which=BOTH, tol: Tol = Tol()):
    """abft_verify (§8 row a2): per-tile status dict {(I,J): bits} and
    counts [tiles_flagged, cols_flagged, rows_flagged, nonfinite_tiles]."""
    status, counts = {}, [0, 0, 0, 0]
    for I, J in tiles:
        tc = check_tile(st, I, J, tiles.view(I, J), which, tol)
        s = tc.status
        status[(I, J)] = s
        if tol.refresh:
            _refresh(st, tc, which)
        if s & (ST_COL | ST_ROW):
            counts[0] += 1
        counts[1] += len(tc.Fc)
        counts[2] += len(tc.Fr)
        counts[3] += 1 if tc.nonfinite else 0
    return status, counts


def _refresh(st: State, tc: TileCheck, which):
    """Reading c-6 'refresh': every UNFLAGGED checksum entry of a verified
    tile is rebased on the recomputed value and its magnitude reset to the
    fresh e^T|X| (flagged entries are left for locate/correct).  Without it the
    magnitude bound compounds |T^-1| factors over the iterations of LU/QR and
    the threshold grows until it hides O(1) errors."""
    nb = st.nb
    c, r, mc, mr = encode_tile(tc.X)
    cs = slice(tc.J * nb, (tc.J + 1) * nb)
    rs = slice(tc.I * nb, (tc.I + 1) * nb)
    if which & COL:
        ok = ~(tc.fce | tc.fcw)
        st.colchk[2 * tc.I:2 * tc.I + 2, cs][:, ok] = c[:, ok]
        if st.colmag is not None:
            st.colmag[tc.I, cs][ok] = mc[ok]
    if which & ROW:
        ok = ~(tc.fre | tc.frw)
        st.rowchk[rs, 2 * tc.J:2 * tc.J + 2][ok, :] = r[ok, :]
        if st.rowmag is not None:
            st.rowmag[rs, tc.J][ok] = mr[ok]


# ----------------------------------------------------------------- locate --
def locate_ratio(de, dw, te, tw, nb):
    """Reading c-5 of L122 'round(delta_2,i / delta_1,i) = j': q = dw/de in
    fp64, j = rint(q) (ties to even), accepted only if q is finite,
    |q − j| ≤ 0.25, 1 ≤ j ≤ nb and |dw − j·de| ≤ tw + j·te.  Returns the
    0-based index or None."""
    de, dw = float(de), float(dw)
    if not (np.isfinite(de) and np.isfinite(dw)) or de == 0.0:
        return None
    q = dw / de
    if not np.isfinite(q):
        return None
    j = float(np.rint(q))
    if abs(q - j) > 0.25 or j < 1 or j > nb:
        return None
    if not abs(dw - j * de) <= tw + j * te:
        return None
    return int(j) - 1


def _m_col(st, tc, j, X):
    """Magnitude behind tau for column j: maintained, else fresh from X."""
    if st.colmag is not None and tc.tc is not None and tc._use_mag:
        return st.colmag[tc.I, tc.J * st.nb + j]
    return float(np.sum(np.abs(X[:, j])))


def _m_row(st, tc, i, X):
    if st.rowmag is not None and tc.tr is not None and tc._use_mag:
        return st.rowmag[tc.I * st.nb + i, tc.J]
    return float(np.sum(np.abs(X[i, :])))


def corrected_value_col(X, c_e, i, j):
    """Reading c-4: x_ij <- c_e[j] − Σ_{r≠i} X[r, j] (identical to the paper's
    'add delta_1' in exact arithmetic, L122, but exact for huge x_bad)."""
    col = X[:, j]
    rest = np.sum(np.delete(col, i))
    return c_e - rest


def corrected_value_row(X, r_e, i, j):
    row = X[i, :]
    return r_e - np.sum(np.delete(row, j))


def _confirm_col(st, tc, i, j, tol):
    """c-7 confirmation: tentatively correct (i,j) via column j, then require
    |delta_e| ≤ tau_e and |delta_w| ≤ tau_w of that column."""
    X = tc.X.copy()
    nb = st.nb
    ce, cw = st.colchk[2 * tc.I, tc.J * nb + j], st.colchk[2 * tc.I + 1, tc.J * nb + j]
    X[i, j] = corrected_value_col(X, ce, i, j)
    v1, v2 = weights(nb)
    with np.errstate(invalid="ignore", over="ignore"):
        de = ce - v1 @ X[:, j]
        dw = cw - v2 @ X[:, j]
        t = tol.scale * tau_e(st, _m_col(st, tc, j, X))
        return bool(np.isfinite(de) and np.isfinite(dw) and abs(de) <= t and abs(dw) <= nb * t)


def _confirm_row(st, tc, i, j, tol):
    X = tc.X.copy()
    nb = st.nb
    re_, rw = st.rowchk[tc.I * nb + i, 2 * tc.J], st.rowchk[tc.I * nb + i, 2 * tc.J + 1]
    X[i, j] = corrected_value_row(X, re_, i, j)
    v1, v2 = weights(nb)
    with np.errstate(invalid="ignore", over="ignore"):
        de = re_ - X[i, :] @ v1
        dw = rw - X[i, :] @ v2
        t = tol.scale * tau_e(st, _m_row(st, tc, i, X))
        return bool(np.isfinite(de) and np.isfinite(dw) and abs(de) <= t and abs(dw) <= nb * t)


def locate_col(st, tc, j, tol, has_r):
    """Row of the error in flagged column j: ratio rule (c-5), else the c-7
    fallback (intersection / unique non-finite / largest |x|, confirmed)."""
    nb = st.nb
    i = locate_ratio(tc.dc[0, j], tc.dc[1, j], tc.tc[j], nb * tc.tc[j], nb)
    if i is not None:
        return i if live(tc.view, i, j) else None
    Fc, Fr = tc.Fc, tc.Fr
    if has_r and len(Fc) == 1 and len(Fr) == 1:
        cand = Fr[0]
    else:
        col = tc.X[:, j]
        nf = np.nonzero(~np.isfinite(col))[0]
        if len(nf) == 1:
            cand = int(nf[0])
        elif len(nf) > 1:
            return None
        else:
            cand = int(np.argmax(np.abs(col)))
    if not live(tc.view, cand, j):
        return None
    return cand if _confirm_col(st, tc, cand, j, tol) else None


def locate_row(st, tc, i, tol, has_c):
    nb = st.nb
    j = locate_ratio(tc.dr[i, 0], tc.dr[i, 1], tc.tr[i], nb * tc.tr[i], nb)
    if j is not None:
        return j if live(tc.view, i, j) else None
    Fc, Fr = tc.Fc, tc.Fr
    if has_c and len(Fc) == 1 and len(Fr) == 1:
        cand = Fc[0]
    else:
        row = tc.X[i, :]
        nf = np.nonzero(~np.isfinite(row))[0]
        if len(nf) == 1:
            cand = int(nf[0])
        elif len(nf) > 1:
            return None
        else:
            cand = int(np.argmax(np.abs(row)))
    if not live(tc.view, i, cand):
        return None
    return cand if _confirm_row(st, tc, i, cand, tol) else None


# ------------------------------------------------------- classify & correct --
def _write(st, I, J, view, i, j, value):
    si, sj = stored_index(view, i, j)
    gi, gj = I * st.nb + si, J * st.nb + sj
    before = float(st.A[gi, gj])
    st.A[gi, gj] = value
    return gi, gj, before


def _reencode_col(st, tc, j, cls, fixes):
    X = tile_view(st.A, tc.I, tc.J, st.nb, tc.view)
    c, _, mc, _ = encode_tile(X)
    g = tc.J * st.nb + j
    before = float(st.colchk[2 * tc.I, g])
    st.colchk[2 * tc.I:2 * tc.I + 2, g] = c[:, j]
    if st.colmag is not None:
        st.colmag[tc.I, g] = mc[j]
    fixes.append(Fix(tc.I, g, before, float(c[0, j]), cls, FIX_COLCHK))


def _reencode_row(st, tc, i, cls, fixes):
    X = tile_view(st.A, tc.I, tc.J, st.nb, tc.view)
    _, r, _, mr = encode_tile(X)
    g = tc.I * st.nb + i
    before = float(st.rowchk[g, 2 * tc.J])
    st.rowchk[g, 2 * tc.J:2 * tc.J + 2] = r[i, :]
    if st.rowmag is not None:
        st.rowmag[g, tc.J] = mr[i]
    fixes.append(Fix(g, tc.J, before, float(r[i, 0]), cls, FIX_ROWCHK))


def _fix_via_col(st, tc, i, j, cls, fixes):
    ce = st.colchk[2 * tc.I, tc.J * st.nb + j]
    new = corrected_value_col(tc.X, ce, i, j)
    gi, gj, before = _write(st, tc.I, tc.J, tc.view, i, j, new)
    fixes.append(Fix(gi, gj, before, float(new), cls))


def _fix_via_row(st, tc, i, j, cls, fixes):
    re_ = st.rowchk[tc.I * st.nb + i, 2 * tc.J]
    new = corrected_value_row(tc.X, re_, i, j)
    gi, gj, before = _write(st, tc.I, tc.J, tc.view, i, j, new)
    fixes.append(Fix(gi, gj, before, float(new), cls))


def classify_fix_round(st, tc, which, tol, fixes):
    """One classify-and-fix round of reading c-11 (combining L122, L145
    'tolerate an erroneous row or column checksum', L330–L334 0D/1D/2D and
    L434 'same row ⇒ 1D, otherwise 2D').  Returns the class applied, CLS_CLEAN
    when nothing is flagged, CLS_2D when nothing applies."""
    has_c, has_r = bool(which & COL), bool(which & ROW)
    Fc, Fr = tc.Fc, tc.Fr
    if not Fc and not Fr:
        return CLS_CLEAN
    sym = tc.view == SYM_LOWER
    # step 3 — all flagged columns locate the same row i (0D / 1D_ROW)
    loc_c = {}
    if has_c and Fc:
        loc_c = {j: locate_col(st, tc, j, tol, has_r) for j in Fc}
        vals = set(loc_c.values())
        if None not in vals and len(vals) == 1:
            i = vals.pop()
            if not has_r or set(Fr) <= {i}:
                cls = CLS_0D if len(Fc) == 1 else CLS_1D_ROW
                for j in Fc:
                    _fix_via_col(st, tc, i, j, cls, fixes)
                return cls
    # step 4 — all flagged rows locate the same column j (0D / 1D_COL)
    if has_r and Fr:
        loc_r = {i: locate_row(st, tc, i, tol, has_c) for i in Fr}
        vals = set(loc_r.values())
        if None not in vals and len(vals) == 1:
            j = vals.pop()
            if not has_c or set(Fc) <= {j}:
                cls = CLS_0D if len(Fr) == 1 else CLS_1D_COL
                for i in Fr:
                    _fix_via_row(st, tc, i, j, cls, fixes)
                return cls
    # step 2 — a lone e- or w-entry that no consistent data location explains
    # (steps 3 and 4 failed): the checksum entry itself is corrupt.  After
    # steps 3-4 (reading c-11b): a data error in local column j changes
    # delta_w by j*delta_e, so for small j it can pass tau_w = nb*tau_e while
    # delta_e fails tau_e; re-encoding then absorbed a locatable data error.
    repaired = False
    if has_c and Fc and (not has_r or not Fr):
        for j in Fc:
            if bool(tc.fce[j]) != bool(tc.fcw[j]):
                _reencode_col(st, tc, j, CLS_CHK_CORRUPT, fixes)
                repaired = True
    if has_r and Fr and (not has_c or not Fc):
        for i in Fr:
            if bool(tc.fre[i]) != bool(tc.frw[i]):
                _reencode_row(st, tc, i, CLS_CHK_CORRUPT, fixes)
                repaired = True
    if repaired:
        return CLS_CHK_CORRUPT
    if sym and has_c:
        # step 5 — SYM_LOWER mirrored pair: one stored element seen twice
        if len(Fc) == 2:
            p, q = Fc
            if loc_c.get(q) == p and loc_c.get(p) == q:
                _fix_via_col(st, tc, p, q, CLS_0D, fixes)
                return CLS_0D
        # step 6 — SYM_CROSS: a corrupted stored row r seen as a cross
        if len(Fc) >= 2:
            for r in Fc:
                others = [j for j in Fc if j != r]
                if all(loc_c.get(j) == r for j in others):
                    for j in others:
                        _fix_via_col(st, tc, r, j, CLS_SYM_CROSS, fixes)
                    return CLS_SYM_CROSS
    # step 5b — one side vouches for the data: the other side is stale (it was
    # updated with a corrupted operand and the data has since been fixed
    # through the good side).  Only after steps 3-6 failed, so a genuine
    # 1D error seen by one side is always corrected first.
    if has_c and has_r:
        if Fr and not Fc:
            for i in Fr:
                _reencode_row(st, tc, i, CLS_STALE_R, fixes)
            return CLS_STALE_R
        if Fc and not Fr:
            for j in Fc:
                _reencode_col(st, tc, j, CLS_STALE_C, fixes)
            return CLS_STALE_C
    return CLS_2D  # step 7


MAX_ROUNDS = 3


def locate_correct_tile(st, I, J, view, which, tol: Tol = Tol()):
    """abft_locate_correct for one tile: ≤3 verify→classify→fix rounds, a
    residual after the last round is 2D (reading c-11).  Returns
    (final_class, fixes); final_class CLS_CLEAN or CLS_2D."""
    fixes = []
    for _ in range(MAX_ROUNDS):
        tc = _checked(st, I, J, view, which, tol)
        cls = classify_fix_round(st, tc, which, tol, fixes)
        if cls == CLS_CLEAN:
            return CLS_CLEAN, fixes
        if cls == CLS_2D:
            return CLS_2D, fixes
    tc = _checked(st, I, J, view, which, tol)
    return (CLS_CLEAN if not tc.Fc and not tc.Fr else CLS_2D), fixes


def _checked(st, I, J, view, which, tol):
    tc = check_tile(st, I, J, view, which, tol)
    tc._use_mag = tol.kind == TOL_MAGNITUDE and st.colmag is not None
    return tc


def locate_correct(st: State, tiles: Tiles, which=BOTH, tol: Tol = Tol()):
    """Every flagged tile of the range: returns (status dict, fixes, counts)
    with counts [tiles_fixed, data_elements_fixed, checksums_repaired,
    uncorrectable_tiles]."""
    status, fixes, counts = {}, [], [0, 0, 0, 0]
    for I, J in tiles:
        view = tiles.view(I, J)
        tc = _checked(st, I, J, view, which, tol)
        if not tc.status & (ST_COL | ST_ROW):
            status[(I, J)] = 0
            continue
        cls, fx = locate_correct_tile(st, I, J, view, which, tol)
        fixes.extend(fx)
        if cls == CLS_2D:
            status[(I, J)] = ST_UNCORRECTABLE
            counts[3] += 1
        else:
            status[(I, J)] = 0
            counts[0] += 1
        counts[1] += sum(1 for f in fx if f.kind == FIX_DATA)
        counts[2] += sum(1 for f in fx if f.kind != FIX_DATA)
    return status, fixes, counts


# ----------------------------------------------------------- margin policy --
def margin_band(st: State, I, J, view, j_local, delta, tol: Tol = Tol(), which_dir="col", idx=None):
    """Reading c-10 ('significant enough bits', L540): for an injected change
    Δ in tile column j, MUST if |Δ| ≥ 16·nb·tau_e[j], NEED-NOT if
    |Δ| ≤ tau_e[j]/8, GRAY otherwise (tau on the error-free state)."""
    X = tile_view(st.A, I, J, st.nb, view)
    if tol.kind == TOL_MAGNITUDE and st.colmag is not None:
        m = st.colmag[I, J * st.nb + j_local]
    else:
        m = float(np.sum(np.abs(X[:, j_local])))
    t = tol.scale * tau_e(st, m)
    a = abs(delta)
    if not np.isfinite(delta) or a >= 16 * st.nb * t:
        return "MUST"
    if a <= t / 8:
        return "NEED_NOT"
    return "GRAY"
