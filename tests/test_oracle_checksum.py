"""Pins of the oracle's checksum core (oracle/checksum.py) against facts that
do not come from the oracle itself: closed forms, exact integer arithmetic
(brute force in Python ints), the correctly rounded math.fsum, and hand-built
fault scenarios whose answer is known by construction.  CPU only."""
import math

import numpy as np
import pytest

import synth_inputs as si
from oracle import checksum as ck


def _int_checksums(Xint):
    """Brute force in Python integers: c_e[j], c_w[j], r_e[i], r_w[i]."""
    nb = len(Xint)
    ce = [sum(Xint[i][j] for i in range(nb)) for j in range(nb)]
    cw = [sum((i + 1) * Xint[i][j] for i in range(nb)) for j in range(nb)]
    re = [sum(Xint[i][j] for j in range(nb)) for i in range(nb)]
    rw = [sum((j + 1) * Xint[i][j] for j in range(nb)) for i in range(nb)]
    return ce, cw, re, rw


@pytest.mark.parametrize("nb", [1, 4, 32, 64])
def test_ones_tile_closed_form(nb):
    # c_e = nb, c_w = nb(nb+1)/2 for every column; rows the same (L108 weights)
    c, r, mc, mr = ck.encode_tile(np.ones((nb, nb)))
    assert np.all(c[0] == nb) and np.all(c[1] == nb * (nb + 1) // 2)
    assert np.all(r[:, 0] == nb) and np.all(r[:, 1] == nb * (nb + 1) // 2)
    assert np.all(mc == nb) and np.all(mr == nb)


@pytest.mark.parametrize("i,j", [(0, 0), (3, 7), (31, 0), (0, 31), (17, 17)])
def test_impulse_tile_closed_form(i, j):
    # X = e_i e_j^T: c[:, j] = (1, i+1), r[i, :] = (1, j+1), zero elsewhere
    nb = 32
    X = np.zeros((nb, nb))
    X[i, j] = 1.0
    c, r, _, _ = ck.encode_tile(X)
    expect_c = np.zeros((2, nb))
    expect_c[:, j] = (1, i + 1)
    expect_r = np.zeros((nb, 2))
    expect_r[i, :] = (1, j + 1)
    assert np.array_equal(c, expect_c) and np.array_equal(r, expect_r)


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("nb", [8, 32, 128])
def test_integer_tile_exact(seed, nb):
    X = si.integers(nb, seed=seed, R=1000)
    c, r, _, _ = ck.encode_tile(X)
    ce, cw, re, rw = _int_checksums([[int(v) for v in row] for row in X])
    assert c[0].tolist() == ce and c[1].tolist() == cw
    assert r[:, 0].tolist() == re and r[:, 1].tolist() == rw


def test_random_tile_within_gamma_of_fsum():
    nb = 256
    X = si.general(nb, seed=3)
    c, r, mc, _ = ck.encode_tile(X)
    g = ck.gamma(nb, ck.unit_roundoff("f64"))
    for j in range(nb):
        exact_e = math.fsum(X[:, j])
        exact_w = math.fsum((i + 1) * X[i, j] for i in range(nb))
        assert abs(c[0, j] - exact_e) <= g * mc[j]
        assert abs(c[1, j] - exact_w) <= g * nb * mc[j]
        assert mc[j] == pytest.approx(math.fsum(abs(x) for x in X[:, j]), rel=1e-14)


def test_views_by_loops():
    nb = 16
    A = si.integers(2 * nb, seed=7)
    I = J = 1
    B = A[nb:2 * nb, nb:2 * nb]
    for view, f in [
        (ck.LOWER, lambda i, j: B[i, j] if i >= j else 0.0),
        (ck.UNIT_LOWER, lambda i, j: B[i, j] if i > j else (1.0 if i == j else 0.0)),
        (ck.UPPER, lambda i, j: B[i, j] if i <= j else 0.0),
        (ck.SYM_LOWER, lambda i, j: B[max(i, j), min(i, j)]),
    ]:
        X = ck.tile_view(A, I, J, nb, view)
        ref = np.array([[f(i, j) for j in range(nb)] for i in range(nb)])
        assert np.array_equal(X, ref)
    # off-diagonal tiles are GENERAL whatever diag_view says
    t = ck.Tiles(0, 2, 0, 2, lower_only=True, diag_view=ck.SYM_LOWER)
    assert list(t) == [(0, 0), (1, 0), (1, 1)]
    assert t.view(1, 0) == ck.GENERAL and t.view(1, 1) == ck.SYM_LOWER


def test_sym_view_row_checksum_is_transposed_column_checksum():
    # L189: for a symmetric block r(A) = c(A)^T
    X = ck.tile_view(si.integers(32, seed=1), 0, 0, 32, ck.SYM_LOWER)
    c, r, mc, mr = ck.encode_tile(X)
    assert np.array_equal(c.T, r) and np.array_equal(mc, mr)


def test_gamma_closed_form():
    u = ck.unit_roundoff("f64")
    assert u == 2.0 ** -53
    assert ck.gamma(512, u) == pytest.approx(512 * u / (1 - 512 * u), rel=0)
    assert ck.unit_roundoff("f32") == 2.0 ** -24


# ----------------------------------------------------------------- verify --
def _state(A, nb, mags=True, view=ck.GENERAL, prec="f64"):
    st = ck.State.alloc(A, nb, prec=prec, mags=mags)
    ck.encode(st, ck.Tiles(0, st.mt, 0, st.nt, diag_view=view))
    return st


def test_verify_integer_matrix_zero_delta():
    st = _state(si.integers(128, seed=2), 32)
    for I, J in ck.Tiles(0, 4, 0, 4):
        tc = ck.check_tile(st, I, J, ck.GENERAL, ck.BOTH)
        assert np.all(tc.dc == 0) and np.all(tc.dr == 0) and tc.status == 0


def test_verify_flags_single_error_exactly():
    st = _state(si.general(128, seed=4), 32)
    st.A[37, 70] += 1.0  # tile (1, 2), local (5, 6)
    status, counts = ck.verify(st, ck.Tiles(0, 4, 0, 4))
    assert {k for k, v in status.items() if v} == {(1, 2)}
    assert counts == [1, 1, 1, 0]
    tc = ck.check_tile(st, 1, 2, ck.GENERAL, ck.BOTH)
    assert tc.Fc == [6] and tc.Fr == [5]
    # delta_e = -1 (maintained − recomputed), delta_w = −(i+1)
    assert tc.dc[0, 6] == pytest.approx(-1.0, abs=1e-12)
    assert tc.dc[1, 6] == pytest.approx(-6.0, abs=1e-12)


@pytest.mark.parametrize("q,expect", [(6.0, 5), (6.2, 5), (6.3, None), (0.0, None), (33.0, None), (32.0, 31)])
def test_locate_ratio_acceptance(q, expect):
    # reading c-5: |q − rint(q)| ≤ 0.25 and 1 ≤ j ≤ nb
    de = 1.0
    dw = q * de
    te = 1.0  # generous consistency slack so only the 0.25 / range rules decide
    assert ck.locate_ratio(de, dw, te, 32 * te, 32) == expect


def test_locate_ratio_consistency_rule():
    # |dw − j·de| must be within tau_w + j·tau_e (reading c-5)
    assert ck.locate_ratio(1.0, 6.1, 1e-3, 32e-3, 32) is None
    assert ck.locate_ratio(1.0, 6.0 + 1e-4, 1e-3, 32e-3, 32) == 5
    assert ck.locate_ratio(0.0, 1.0, 1.0, 1.0, 32) is None
    assert ck.locate_ratio(np.nan, 1.0, 1.0, 1.0, 32) is None


# ------------------------------------------------------ locate / classify --
def _fix_all(st, view=ck.GENERAL, which=ck.BOTH):
    t = ck.Tiles(0, st.mt, 0, st.nt, lower_only=(view == ck.SYM_LOWER), diag_view=view)
    return ck.locate_correct(st, t, which)


def test_0d_integer_fix_is_exact():
    A = si.integers(64, seed=5)
    st = _state(A, 32)
    st.A[40, 3] = 1e6
    status, fixes, counts = _fix_all(st)
    assert counts == [1, 1, 0, 0]
    assert [(f.gi, f.gj, f.cls) for f in fixes] == [(40, 3, ck.CLS_0D)]
    assert np.array_equal(st.A, A)


@pytest.mark.parametrize("bit", [62, 63, 61, 55, 40])
def test_exponent_and_sign_flips_fixed(bit):
    A = si.general(64, seed=6)
    st = _state(A, 32)
    st.A[10, 20] = si.flip_bits(A[10, 20], [bit])
    _, fixes, counts = _fix_all(st)
    assert counts[3] == 0 and len(fixes) == 1 and (fixes[0].gi, fixes[0].gj) == (10, 20)
    assert abs(st.A[10, 20] - A[10, 20]) <= 64 * ck.unit_roundoff("f64") * np.abs(A[:32, 20]).sum()


@pytest.mark.parametrize("value", [np.inf, -np.inf, np.nan, 1e308, -1e300])
def test_nonfinite_and_huge_values_fixed(value):
    # reading c-7: non-finite / overflowing residual → fallback + confirmation
    A = si.general(64, seed=8)
    st = _state(A, 32)
    st.A[33, 40] = value
    _, fixes, counts = _fix_all(st)
    assert counts[3] == 0 and [(f.gi, f.gj) for f in fixes] == [(33, 40)]
    assert st.A[33, 40] == pytest.approx(A[33, 40], abs=1e-12)


def test_1d_row_error():
    # a corrupted row segment inside a tile (on-chip TMU fault, L359) → 1D_ROW
    A = si.general(64, seed=9)
    st = _state(A, 32)
    st.A[35, 32:40] += np.arange(1, 9)
    _, fixes, counts = _fix_all(st)
    assert counts == [1, 8, 0, 0]
    assert {f.cls for f in fixes} == {ck.CLS_1D_ROW}
    assert np.allclose(st.A, A, atol=1e-12)


def test_1d_col_error():
    A = si.general(64, seed=10)
    st = _state(A, 32)
    st.A[0:32:3, 50] -= 3.0
    _, fixes, counts = _fix_all(st)
    assert counts[3] == 0 and {f.cls for f in fixes} == {ck.CLS_1D_COL}
    assert np.allclose(st.A, A, atol=1e-12)


def test_1d_row_in_column_checksum_only_tile():
    # column panel after PU keeps c only (L139, c-9); 1D row → fixable (L434)
    A = si.general(64, seed=11)
    st = _state(A, 32)
    st.A[7, 0:32:2] *= -3.0
    _, fixes, counts = _fix_all(st, which=ck.COL)
    assert counts[3] == 0 and {f.cls for f in fixes} == {ck.CLS_1D_ROW}
    assert np.allclose(st.A, A, atol=1e-12)


def test_2d_error_is_uncorrectable():
    # two errors in different rows and columns of one c-only tile (L434)
    A = si.general(64, seed=12)
    st = _state(A, 32)
    st.A[3, 4] += 5.0
    st.A[9, 11] += 7.0
    status, _, counts = _fix_all(st, which=ck.COL)
    assert counts[3] == 1 and status[(0, 0)] == ck.ST_UNCORRECTABLE


@pytest.mark.parametrize("w", [0, 1])
def test_checksum_corrupt_entry_repaired(w):
    # L145: full checksums tolerate an erroneous checksum
    A = si.general(64, seed=13)
    st = _state(A, 32)
    st.colchk[2 * 1 + w, 45] += 100.0
    _, fixes, counts = _fix_all(st)
    assert counts[3] == 0 and [f.cls for f in fixes] == [ck.CLS_CHK_CORRUPT]
    assert fixes[0].kind == ck.FIX_COLCHK and np.array_equal(st.A, A)
    assert ck.verify(st, ck.Tiles(0, 2, 0, 2))[1][0] == 0


def _absorbed_column_damage(seed):
    """A column of data errors that the column checksums absorbed (the TMU's
    c-rule ran on the corrupted operand): tile (1, 1), local column 0
    (weight 1), half of the rows off by 1e-12 (above tau_e ~ 1e-13 of this
    U(-1,1) nb=32 tile but below tau_w = nb tau_e: delta_w = 1 * delta_e
    flags e only), the other half by 0.5 (both flagged)."""
    A = si.general(64, seed=seed)
    st = _state(A, 32)
    d = np.where(np.arange(32) % 2 == 0, 1e-12, 0.5) * (1 + np.arange(32) / 32)
    st.A[32:64, 32] += d
    X = st.A[32:64, 32:64]
    st.colchk[2:4, 32] = [X[:, 0].sum(), (np.arange(1, 33) * X[:, 0]).sum()]  # absorbed
    st.colmag[1, 32] = np.abs(X[:, 0]).sum()
    return A, st, d


def test_e_only_row_flags_that_locate_are_data_errors():
    """Reading c-11b: rows flagged by e only whose ratio locates local column
    0 are data errors (1D_COL through the rows), not corrupt row checksums;
    by construction the original matrix comes back and no checksum entry is
    declared corrupt."""
    A, st, d = _absorbed_column_damage(16)
    status, fixes, counts = _fix_all(st)
    assert counts[3] == 0
    cls = {f.cls for f in fixes}
    assert ck.CLS_CHK_CORRUPT not in cls and ck.CLS_1D_COL in cls, cls
    assert sum(f.cls == ck.CLS_1D_COL for f in fixes) == 32
    assert np.abs(st.A - A).max() <= 1e-14 and np.abs(st.A - A).max() < d.min() / 10
    assert ck.verify(st, ck.Tiles(0, 2, 0, 2))[1][0] == 0


def test_stale_row_checksum():
    # data consistent with c, r disagrees in two rows → STALE_R (reading c-11 5b)
    A = si.general(64, seed=14)
    st = _state(A, 32)
    st.rowchk[5, 0] += 2.0
    st.rowchk[5, 1] += 11.0
    st.rowchk[9, 0] += 3.0
    st.rowchk[9, 1] += 7.0
    _, fixes, counts = _fix_all(st)
    assert {f.cls for f in fixes} == {ck.CLS_STALE_R} and np.array_equal(st.A, A)
    assert counts[3] == 0


def test_stale_column_checksum():
    A = si.general(64, seed=15)
    st = _state(A, 32)
    st.colchk[0, 3] += 2.0
    st.colchk[1, 3] += 3.3
    st.colchk[0, 5] += 1.0
    st.colchk[1, 5] += 2.7
    _, fixes, counts = _fix_all(st)
    assert {f.cls for f in fixes} == {ck.CLS_STALE_C} and np.array_equal(st.A, A)


def test_sym_lower_mirrored_pair():
    # one stored error below the diagonal appears twice in the symmetric view
    A = si.spd(64, seed=16)
    st = _state(A, 32, view=ck.SYM_LOWER)
    st.A[20, 4] += 9.0
    _, fixes, counts = _fix_all(st, view=ck.SYM_LOWER)
    assert [(f.gi, f.gj, f.cls) for f in fixes] == [(20, 4, ck.CLS_0D)]
    assert np.allclose(np.tril(st.A), np.tril(A), atol=1e-12)


def test_sym_lower_diagonal_element():
    A = si.spd(64, seed=17)
    st = _state(A, 32, view=ck.SYM_LOWER)
    st.A[40, 40] *= 4.0
    _, fixes, counts = _fix_all(st, view=ck.SYM_LOWER)
    assert [(f.gi, f.gj, f.cls) for f in fixes] == [(40, 40, ck.CLS_0D)]


def test_sym_cross():
    # stored row r of a diagonal SYRK tile corrupted (left of and below the
    # diagonal): a cross in the symmetric view → SYM_CROSS then 0D (c-11 step 6)
    A = si.spd(32, seed=18)
    st = _state(A, 32, view=ck.SYM_LOWER)
    r = 9
    st.A[r, :r] += np.linspace(1, 2, r)
    st.A[r + 1:, r] += np.linspace(3, 4, 32 - r - 1)
    st.A[r, r] += 5.0
    _, fixes, counts = _fix_all(st, view=ck.SYM_LOWER)
    assert counts[3] == 0
    assert ck.CLS_SYM_CROSS in {f.cls for f in fixes}
    assert np.allclose(np.tril(st.A), np.tril(A), atol=1e-10)


def test_posteriori_tolerance_without_magnitude_arrays():
    A = si.general(64, seed=19)
    st = _state(A, 32, mags=False)
    st.A[1, 1] += 1.0
    _, fixes, counts = _fix_all(st)
    assert [(f.gi, f.gj) for f in fixes] == [(1, 1)]


# ---------------------------------------------------- brute force (c-10) --
@pytest.mark.parametrize("prec", ["f64", "f32"])
def test_brute_force_single_flips_one_tile(prec):
    """Every element × every bit of one off-diagonal tile (nb=16): MUST-band
    flips are detected, located and corrected; NEED-NOT flips are not flagged
    (reading c-10 of 'significant enough bits', L540)."""
    nb = 16
    dt = np.float64 if prec == "f64" else np.float32
    nbits = 64 if prec == "f64" else 32
    A0 = si.spd(2 * nb, seed=20).astype(dt).astype(np.float64)
    base = _state(A0, nb, prec=prec)
    I, J = 1, 0
    n_must = n_need = 0
    for i in range(nb):
        for j in range(nb):
            gi, gj = I * nb + i, J * nb + j
            for b in range(nbits):
                new = si.flip_bits(A0[gi, gj], [b], dt)
                delta = new - A0[gi, gj] if np.isfinite(new) else np.inf
                band = ck.margin_band(base, I, J, ck.GENERAL, j, delta)
                if band == "GRAY":
                    continue
                st = base.copy()
                st.A[gi, gj] = new
                tc = ck.check_tile(st, I, J, ck.GENERAL, ck.BOTH)
                if band == "NEED_NOT":
                    n_need += 1
                    assert tc.status == 0, (i, j, b)
                    continue
                n_must += 1
                cls, fixes = ck.locate_correct_tile(st, I, J, ck.GENERAL, ck.BOTH)
                assert cls == ck.CLS_CLEAN, (i, j, b)
                assert [(f.gi, f.gj) for f in fixes if f.kind == ck.FIX_DATA] == [(gi, gj)], (i, j, b)
                tol = 16 * nb * ck.unit_roundoff(prec) * base.colmag[I, gj]
                assert abs(st.A[gi, gj] - A0[gi, gj]) <= tol, (i, j, b)
    assert n_must > 0 and n_need > 0
