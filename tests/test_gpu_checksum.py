"""GPU parity of the checksum hot path (§8 rows a1–a3) against the oracle,
called through the C ABI (ctypes binding)."""
import numpy as np
import pytest
import torch

import synth_inputs as si
from oracle import checksum as ck
from tests.gpu_helpers import dev, gpu_state_to_oracle, host, normwise_err

pytestmark = pytest.mark.gpu

TOL = {"f64": 1e-12, "f32": 1e-5}
TDT = {"f64": torch.float64, "f32": torch.float32}
NDT = {"f64": np.float64, "f32": np.float32}


def _encode(lib, A_np, nb, prec="f64", view=ck.GENERAL, lower_only=False, which=ck.BOTH, mags=True, ld=None):
    A = dev(A_np, TDT[prec], ld=ld)
    mat = lib.Mat.alloc(A, nb, mags=mags)
    t = lib.tiles(0, mat.mt, 0, mat.nt, lower_only, view)
    lib.abft_encode(mat, t, which)
    torch.cuda.synchronize()
    return mat, t


def _oracle_state(A_np, nb, prec="f64", view=ck.GENERAL, lower_only=False, which=ck.BOTH, mags=True):
    A64 = A_np.astype(NDT[prec]).astype(np.float64)
    st = ck.State.alloc(A64, nb, prec=prec, mags=mags)
    ck.encode(st, ck.Tiles(0, st.mt, 0, st.nt, lower_only, view), which)
    return st


def _compare_encode(mat, st, prec, lower_only=False, view=ck.GENERAL, exact=False):
    g = gpu_state_to_oracle(mat, prec)
    nb = st.nb
    worst = 0.0
    for I, J in ck.Tiles(0, st.mt, 0, st.nt, lower_only, view):
        v = view if I == J else ck.GENERAL
        X = ck.tile_view(st.A, I, J, nb, v)
        cs, rs = slice(J * nb, (J + 1) * nb), slice(I * nb, (I + 1) * nb)
        cg, cr = g.colchk[2 * I:2 * I + 2, cs], st.colchk[2 * I:2 * I + 2, cs]
        rg, rr = g.rowchk[rs, 2 * J:2 * J + 2], st.rowchk[rs, 2 * J:2 * J + 2]
        if exact:
            assert np.array_equal(cg, cr) and np.array_equal(rg, rr), (I, J)
            assert np.array_equal(g.colmag[I, cs], st.colmag[I, cs])
        worst = max(worst, normwise_err(cg, cr, X, 0), normwise_err(rg, rr, X, 1))
        mag_err = np.abs(g.colmag[I, cs] - st.colmag[I, cs]) / np.maximum(st.colmag[I, cs], 1e-300)
        worst = max(worst, float(mag_err.max()))
    assert worst <= TOL[prec], worst
    return worst


@pytest.mark.parametrize("prec", ["f64", "f32"])
@pytest.mark.parametrize("nb", [32, 64, 128, 256, 512, 1024])
def test_encode_integer_bit_exact(lib, prec, nb):
    n = 2 * nb if nb >= 512 else 4 * nb
    A = si.integers(n, seed=nb, R=8 if prec == "f32" else 1000)
    mat, _ = _encode(lib, A, nb, prec)
    st = _oracle_state(A, nb, prec)
    _compare_encode(mat, st, prec, exact=True)


@pytest.mark.parametrize("prec", ["f64", "f32"])
@pytest.mark.parametrize("nb,m,n", [(32, 256, 256), (64, 192, 320), (128, 384, 256), (256, 512, 768),
                                    (512, 1024, 1536), (1024, 2048, 1024)])
def test_encode_random_normwise(lib, prec, nb, m, n):
    A = si.general(m, n, seed=m + n)
    mat, _ = _encode(lib, A, nb, prec)
    st = _oracle_state(A, nb, prec)
    _compare_encode(mat, st, prec)


@pytest.mark.parametrize("view", [ck.SYM_LOWER, ck.LOWER, ck.UNIT_LOWER, ck.UPPER])
@pytest.mark.parametrize("nb", [32, 256, 1024])
def test_encode_diag_views(lib, view, nb):
    n = 2 * nb
    A = si.spd(n, seed=3) if view == ck.SYM_LOWER else si.general(n, seed=3)
    lower = view == ck.SYM_LOWER
    mat, _ = _encode(lib, A, nb, "f64", view=view, lower_only=lower)
    st = _oracle_state(A, nb, "f64", view=view, lower_only=lower)
    _compare_encode(mat, st, "f64", lower_only=lower, view=view)


def test_encode_odd_leading_dimension(lib):
    # lda*8 not a multiple of 16 -> the non-TMA staging path
    A = si.general(256, seed=4)
    mat, _ = _encode(lib, A, 64, "f64", ld=257)
    assert mat.A.stride(1) == 257
    st = _oracle_state(A, 64, "f64")
    _compare_encode(mat, st, "f64")


@pytest.mark.parametrize("prec", ["f64", "f32"])
@pytest.mark.parametrize("nb,n", [(32, 256), (256, 1024), (512, 2048), (1024, 2048), (1024, 4096), (512, 8192)])
def test_verify_after_encode_is_exactly_zero(lib, prec, nb, n):
    """c-27 pin: one deterministic reduction order -> delta == 0 bit-exactly,
    whatever slab split the launcher picks for the tile count."""
    A = si.general(n, seed=nb)
    mat, t = _encode(lib, A, nb, prec)
    rep = lib.Report.alloc(mat, deltas=True)
    lib.abft_verify(mat, t, ck.BOTH, lib.abft_tol_t(ck.TOL_MAGNITUDE, 1.0), rep)
    # a sub-range (different grid / slab split) must also be exact
    sub = lib.tiles(1, mat.mt, 0, 1)
    lib.abft_verify(mat, sub, ck.BOTH, lib.abft_tol_t(ck.TOL_MAGNITUDE, 1.0), rep)
    torch.cuda.synchronize()
    assert torch.count_nonzero(rep.dcol) == 0 and torch.count_nonzero(rep.drow) == 0
    assert torch.count_nonzero(rep.status) == 0 and torch.count_nonzero(rep.counts) == 0


def test_verify_sym_lower_after_encode_is_zero(lib):
    A = si.spd(1024, seed=5)
    mat, t = _encode(lib, A, 256, "f64", view=ck.SYM_LOWER, lower_only=True)
    rep = lib.Report.alloc(mat, deltas=True)
    lib.abft_verify(mat, t, ck.BOTH, lib.abft_tol_t(ck.TOL_MAGNITUDE, 1.0), rep)
    torch.cuda.synchronize()
    assert torch.count_nonzero(rep.status) == 0 and torch.count_nonzero(rep.dcol) == 0


def _fix_tuple_list(fixes):
    return sorted((f[0], f[1], f[4], f[5]) for f in fixes)


def _clone_mat(lib, mat):
    cl = lambda x: None if x is None else x.t().clone().t()  # keep the column-major strides
    return lib.Mat(cl(mat.A), mat.nb, cl(mat.colchk), cl(mat.rowchk), cl(mat.colmag), cl(mat.rowmag))


def _run_locate(lib, mat, t, which, view=ck.GENERAL, tol=None):
    """abft_verify then abft_locate_correct on `mat`; and, on a copy of the
    same corrupted state, the fused abft_check, whose status, counts, fix
    records and corrected arrays must equal the two-launch path's bit for bit."""
    tol = tol or lib.abft_tol_t(ck.TOL_MAGNITUDE, 1.0)
    twin = _clone_mat(lib, mat)
    rep = lib.Report.alloc(mat)
    lib.abft_verify(mat, t, which, tol, rep)
    status_v = host(rep.status.clone()).astype(int)
    fixbuf = torch.zeros(4096 * lib.FIX_BYTES, dtype=torch.uint8, device="cuda")
    nfix = torch.zeros(1, dtype=torch.int32, device="cuda")
    lib.abft_locate_correct(mat, t, which, tol, rep, fixbuf, nfix)
    rep2 = lib.Report.alloc(twin)
    fixbuf2 = torch.zeros_like(fixbuf)
    nfix2 = torch.zeros_like(nfix)
    lib.abft_check(twin, t, which, tol, rep2, fixbuf2, nfix2)
    torch.cuda.synchronize()
    n = int(nfix.item())
    fixes = lib.decode_fixes(fixbuf, n)
    assert int(nfix2.item()) == n
    assert torch.equal(rep.status, rep2.status) and torch.equal(rep.counts, rep2.counts)
    key = lambda f: (f[0], f[1], f[4], f[5], repr(f[2]), repr(f[3]))  # NaN-safe
    assert sorted(map(key, fixes)) == sorted(map(key, lib.decode_fixes(fixbuf2, n)))
    for x, y in [(mat.A, twin.A), (mat.colchk, twin.colchk), (mat.rowchk, twin.rowchk), (mat.colmag, twin.colmag),
                 (mat.rowmag, twin.rowmag)]:
        if x is not None:
            assert torch.equal(x.view(torch.int64 if x.dtype == torch.float64 else torch.int32),
                               y.view(torch.int64 if y.dtype == torch.float64 else torch.int32))
    return status_v, host(rep.status).astype(int), rep.counts.cpu().numpy(), fixes


def _oracle_locate(st, t_or, which):
    status_v, counts_v = ck.verify(st, t_or, which)
    status_f, fixes, counts_f = ck.locate_correct(st, t_or, which)
    return status_v, counts_v, status_f, fixes, counts_f


def _compare_locate(lib, A_np, nb, mutate, which=ck.BOTH, view=ck.GENERAL, lower_only=False, prec="f64"):
    """Apply the same corruption on both sides; flags, classes, positions must
    agree exactly; corrected data within the fp64 / fp32 tolerance (fp32: the
    oracle sums the fp32 values in fp64, the GPU in fp32; outside the GRAY
    band of c-10 every decision is the same)."""
    A_np = A_np.astype(NDT[prec]).astype(np.float64)
    mat, t = _encode(lib, A_np, nb, prec, view=view, lower_only=lower_only)
    st = _oracle_state(A_np, nb, prec, view=view, lower_only=lower_only)
    mutate(st, mat)
    torch.cuda.synchronize()
    sv, sf, counts, fixes = _run_locate(lib, mat, t, which, view)
    t_or = ck.Tiles(0, st.mt, 0, st.nt, lower_only, view)
    osv, ocv, osf, ofixes, ocf = _oracle_locate(st, t_or, which)
    # fp32: ST_NONFINITE / counts[3] record fp32 overflow of the recomputed
    # sums, which the oracle (fp32 data summed in fp64, c-21) cannot see
    nfm = ~ck.ST_NONFINITE if prec == "f32" else -1
    for (I, J), s in osv.items():
        assert sv[I, J] & nfm == s & nfm, ((I, J), sv[I, J], s)
    if prec == "f32":
        counts[3], ocv = 0, ocv[:3] + [0]
    assert list(counts[:4]) == ocv, (counts, ocv)
    for (I, J), s in osf.items():
        assert sf[I, J] == s, ((I, J), sf[I, J], s)
    assert list(counts[4:]) == ocf, (counts[4:], ocf)
    assert _fix_tuple_list(fixes) == sorted((f.gi, f.gj, f.cls, f.kind) for f in ofixes)
    g = gpu_state_to_oracle(mat, prec)
    scale = np.abs(st.A[np.isfinite(st.A)]).max()
    assert np.abs(g.A - st.A).max() <= TOL[prec] * scale
    return fixes


def _set(st, mat, i, j, value):
    value = float(np.asarray(value, dtype=np.float32)) if mat.A.dtype == torch.float32 else value
    st.A[i, j] = value
    mat.A[i, j] = value


@pytest.mark.parametrize("prec", ["f64", "f32"])
def test_locate_0d_every_tile_config1(lib, prec):
    """BASELINE configs[0] shape: fp64 SPD n=256 nb=32, one MUST-band flip in
    every lower tile (paper L275: one fault per block between checks)."""
    nb, n = 32, 256
    A = si.spd(n, seed=0)
    plan = si.random_positions(n // nb, n // nb, nb, seed=1, lower_only=True)
    g = si.rng(2)

    def mutate(st, mat):
        for I, J, i, j in plan:
            gi, gj = I * nb + i, J * nb + j
            if I == J and i < j:
                gi, gj = I * nb + j, J * nb + i  # stored lower element
            if prec == "f64":
                bit = int(g.integers(40, 64))
                _set(st, mat, gi, gj, si.flip_bits(A[gi, gj], [bit]))
            else:  # fp32: bits 20-31 (c-10 MUST band of the fp32 tile)
                bit = int(g.integers(20, 32))
                _set(st, mat, gi, gj, si.flip_bits(np.float32(A[gi, gj]), [bit], np.float32))

    fixes = _compare_locate(lib, A, nb, mutate, view=ck.SYM_LOWER, lower_only=True, prec=prec)
    assert len([f for f in fixes if f[5] == ck.FIX_DATA]) == len(plan)


@pytest.mark.parametrize("prec", ["f64", "f32"])
@pytest.mark.parametrize("case", ["1d_row", "1d_col", "chk_e", "chk_w", "stale_r", "stale_c", "2d", "inf", "nan",
                                  "huge", "absorbed_col"])
def test_locate_classes_match_oracle(lib, case, prec):
    if prec == "f32" and case == "absorbed_col":
        pytest.skip("the c-11b case is built from 1e-12 relative deltas (fp64 only)")
    A = si.general(128, seed=30)
    nb = 64

    def mutate(st, mat):
        if case == "1d_row":
            for j in range(64, 72):
                _set(st, mat, 70, j, A[70, j] + j)
        elif case == "1d_col":
            for i in range(0, 64, 5):
                _set(st, mat, i, 100, A[i, 100] - 3.0)
        elif case in ("chk_e", "chk_w"):
            w = 0 if case == "chk_e" else 1
            st.colchk[2 + w, 10] += 50.0
            mat.colchk[2 + w, 10] += 50.0
        elif case == "stale_r":
            for r, de, dw in [(3, 2.0, 11.0), (9, 3.0, 7.0)]:
                st.rowchk[r, 0] += de
                st.rowchk[r, 1] += dw
                mat.rowchk[r, 0] += de
                mat.rowchk[r, 1] += dw
        elif case == "stale_c":
            for c, de, dw in [(65, 2.0, 3.3), (70, 1.0, 2.7)]:
                st.colchk[0, c] += de
                st.colchk[1, c] += dw
                mat.colchk[0, c] += de
                mat.colchk[1, c] += dw
        elif case == "2d":
            _set(st, mat, 3, 4, A[3, 4] + 5.0)
            _set(st, mat, 9, 11, A[9, 11] + 7.0)
        elif case == "inf":
            _set(st, mat, 33, 40, np.inf)
        elif case == "nan":
            _set(st, mat, 33, 40, np.nan)
        elif case == "huge":
            _set(st, mat, 33, 40, 1e308 if prec == "f64" else 3e38)
        elif case == "absorbed_col":  # c-11b: e-only row flags that locate column 0 are data errors
            d = np.where(np.arange(64) % 2 == 0, 1e-12, 0.5) * (1 + np.arange(64) / 64)
            for i in range(64):
                _set(st, mat, 64 + i, 64, A[64 + i, 64] + d[i])
            x = st.A[64:128, 64]
            ce, cw, cm = x.sum(), (np.arange(1, 65) * x).sum(), np.abs(x).sum()
            st.colchk[2:4, 64] = [ce, cw]
            st.colmag[1, 64] = cm
            mat.colchk[2, 64], mat.colchk[3, 64], mat.colmag[1, 64] = float(ce), float(cw), float(cm)

    _compare_locate(lib, A, nb, mutate, prec=prec)


@pytest.mark.parametrize("prec", ["f64", "f32"])
@pytest.mark.parametrize("which", [ck.COL, ck.ROW])
def test_locate_single_side(lib, which, prec):
    A = si.general(128, seed=31)

    def mutate(st, mat):
        if which == ck.COL:
            for j in range(0, 40, 3):
                _set(st, mat, 20, j, A[20, j] * -2.0)
        else:
            for i in range(64, 128, 7):
                _set(st, mat, i, 90, A[i, 90] + 4.0)

    _compare_locate(lib, A, 64, mutate, which=which, prec=prec)


@pytest.mark.parametrize("prec", ["f64", "f32"])
def test_locate_sym_pair_and_cross(lib, prec):
    A = si.spd(128, seed=32)

    def mutate(st, mat):
        _set(st, mat, 20, 4, A[20, 4] + 9.0)  # mirrored pair in tile (0,0)
        r = 64 + 9  # cross in tile (1,1)
        for j in range(64, r):
            _set(st, mat, r, j, A[r, j] + 1.5)
        for i in range(r + 1, 128):
            _set(st, mat, i, r, A[i, r] + 3.5)
        _set(st, mat, r, r, A[r, r] + 5.0)

    _compare_locate(lib, A, 64, mutate, view=ck.SYM_LOWER, lower_only=True, prec=prec)


def test_inject_is_xor(lib):
    A = dev(si.general(64, seed=1))
    before = A[5, 7].item()
    lib.abft_inject(A, 5, 7, 1 << 62)
    torch.cuda.synchronize()
    assert A[5, 7].item() == si.flip_bits(before, [62])


@pytest.mark.parametrize("prec,n", [("f64", 16384), ("f32", 16384), ("f64", 30720)])
def test_full_size_sampled_tiles(lib, prec, n):
    """BASELINE config-4 sized matrices (n=16384, nb=512) and the bench's own
    launch (fp64 n=30720 nb=512, the metric's size): sampled tiles vs the
    oracle, plus the verify-after-encode invariant over the whole matrix."""
    nb = 512
    A = si.general_device(n, seed=7, dtype=TDT[prec])
    mat = lib.Mat.alloc(A, nb)
    t = lib.tiles(0, n // nb, 0, n // nb)
    lib.abft_encode(mat, t)
    rep = lib.Report.alloc(mat)
    lib.abft_verify(mat, t, ck.BOTH, lib.abft_tol_t(ck.TOL_MAGNITUDE, 1.0), rep)
    torch.cuda.synchronize()
    assert torch.count_nonzero(rep.counts) == 0
    g = si.rng(3)
    for _ in range(6):
        I, J = int(g.integers(0, n // nb)), int(g.integers(0, n // nb))
        X = host(A[I * nb:(I + 1) * nb, J * nb:(J + 1) * nb])
        c, r, mc, mr = ck.encode_tile(X)
        cg = host(mat.colchk[2 * I:2 * I + 2, J * nb:(J + 1) * nb])
        rg = host(mat.rowchk[I * nb:(I + 1) * nb, 2 * J:2 * J + 2])
        assert normwise_err(cg, c, X, 0) <= TOL[prec]
        assert normwise_err(rg, r, X, 1) <= TOL[prec]


# Ranges the launcher cuts into ragged stacks of K tiles (PASS_SEG) plus a
# diagonal-only launch when the diagonal view is masked (PASS_DIAG): lower-only
# triangles, offset sub-ranges, heights K does not divide, masked diagonals
# that split a tile column in two.  (I0, I1, J0, J1, lower_only, view) with
# I1/J1 = None for nt.
SEG_RANGES = [(0, None, 0, None, True, ck.SYM_LOWER), (0, None, 0, None, True, ck.GENERAL),
              (2, None, 1, -2, True, ck.LOWER), (1, -1, 0, 3, False, ck.GENERAL),
              (0, None, 0, None, False, ck.UNIT_LOWER), (3, None, 0, None, False, ck.UPPER)]


def _seg_case(nb):
    nt = 19 if nb <= 64 else (11 if nb == 128 else 7)
    return nt, nt * nb


def _rng(r, nt):
    I0, I1, J0, J1, lower, view = r
    fix = lambda v: nt if v is None else (nt + v if v < 0 else v)  # noqa: E731
    return fix(I0), fix(I1), fix(J0), fix(J1), lower, view


@pytest.mark.parametrize("prec,nb", [("f64", 32), ("f64", 64), ("f64", 128), ("f64", 256), ("f32", 32),
                                     ("f32", 128), ("f32", 256), ("f32", 512)])
@pytest.mark.parametrize("ri", range(len(SEG_RANGES)))
def test_encode_segmented_ranges_bit_exact(lib, prec, nb, ri):
    nt, n = _seg_case(nb)
    I0, I1, J0, J1, lower, view = _rng(SEG_RANGES[ri], nt)
    A = si.integers(n, seed=nb + ri, R=8 if prec == "f32" else 1000)
    if view == ck.SYM_LOWER:
        A = A + A.T
    mat = lib.Mat.alloc(dev(A, TDT[prec]), nb)
    lib.abft_encode(mat, lib.tiles(I0, I1, J0, J1, lower, view))
    torch.cuda.synchronize()
    st = ck.State.alloc(A.astype(np.float64), nb, prec=prec)
    tt = ck.Tiles(I0, I1, J0, J1, lower, view)
    ck.encode(st, tt)
    g = gpu_state_to_oracle(mat, prec)
    seen = set(tt)
    assert seen
    for I in range(nt):
        for J in range(nt):
            cs, rs = slice(J * nb, (J + 1) * nb), slice(I * nb, (I + 1) * nb)
            if (I, J) in seen:  # exact sums of integers: every order gives the same bits
                assert np.array_equal(g.colchk[2 * I:2 * I + 2, cs], st.colchk[2 * I:2 * I + 2, cs]), (I, J)
                assert np.array_equal(g.rowchk[rs, 2 * J:2 * J + 2], st.rowchk[rs, 2 * J:2 * J + 2]), (I, J)
                assert np.array_equal(g.colmag[I, cs], st.colmag[I, cs]), (I, J)
                assert np.array_equal(g.rowmag[rs, J], st.rowmag[rs, J]), (I, J)
            else:  # tiles outside the range are not written
                assert not g.colchk[2 * I:2 * I + 2, cs].any() and not g.rowchk[rs, 2 * J:2 * J + 2].any(), (I, J)


@pytest.mark.parametrize("prec,nb", [("f64", 32), ("f64", 256), ("f32", 64), ("f32", 512)])
def test_verify_segmented_after_rect_encode_is_exactly_zero(lib, prec, nb):
    """c-27 pin across launch shapes: checksums written by a full rectangular
    encode (PASS_RECT stacks) are recomputed bit-identically by the ragged
    PASS_SEG stacks of lower-only / offset / ragged-height verifies."""
    nt, n = _seg_case(nb)
    A = si.general(n, seed=nb)
    mat, _ = _encode(lib, A, nb, prec)
    rep = lib.Report.alloc(mat, deltas=True)
    tol = lib.abft_tol_t(ck.TOL_MAGNITUDE, 1.0)
    for r in SEG_RANGES[1:4]:
        I0, I1, J0, J1, lower, _ = _rng(r, nt)
        lib.abft_verify(mat, lib.tiles(I0, I1, J0, J1, lower, ck.GENERAL), ck.BOTH, tol, rep)
    torch.cuda.synchronize()
    assert torch.count_nonzero(rep.dcol) == 0 and torch.count_nonzero(rep.drow) == 0
    assert torch.count_nonzero(rep.status) == 0 and torch.count_nonzero(rep.counts) == 0


@pytest.mark.parametrize("prec,nb", [("f64", 64), ("f32", 256)])
def test_verify_segmented_flags_every_tile(lib, prec, nb):
    """One MUST-band corruption in every tile of a lower-only SYM range: the
    ragged stacks and the diagonal launch flag exactly those tiles."""
    nt, n = _seg_case(nb)
    A = si.spd(n, seed=9)
    mat, t = _encode(lib, A, nb, prec, view=ck.SYM_LOWER, lower_only=True)
    for I in range(nt):
        for J in range(I + 1):
            i, j = (I * nb + 5, J * nb + 3)
            mat.A[i, j] += 1e3
    rep = lib.Report.alloc(mat)
    lib.abft_verify(mat, t, ck.BOTH, lib.abft_tol_t(ck.TOL_MAGNITUDE, 1.0), rep)
    torch.cuda.synchronize()
    s = host(rep.status)
    for I in range(nt):
        for J in range(nt):
            assert (s[I, J] != 0) == (I >= J), (I, J, s[I, J])
    assert int(rep.counts[0].item()) == nt * (nt + 1) // 2


# ---- f3 baseline: the GEMM-based recalculation (abft_verify_gemm) --------
@pytest.mark.parametrize("prec", ["f64", "f32"])
@pytest.mark.parametrize("rng_case", ["full", "sym_lower", "lower_col"])
def test_verify_gemm_matches_fused(lib, prec, rng_case):
    """The prior-art GEMM recalculation (L442) reaches the same verdicts as the
    fused pass: identical tile status and counts on MUST-band corruptions, and
    deltas equal within the normwise tolerance of c-1."""
    nb, n = 64, 384
    A = si.spd(n, seed=12) if rng_case != "full" else si.general(n, seed=12)
    view = {"full": ck.GENERAL, "sym_lower": ck.SYM_LOWER, "lower_col": ck.LOWER}[rng_case]
    lower = rng_case != "full"
    which = ck.COL if rng_case == "lower_col" else ck.BOTH
    mat, t = _encode(lib, A, nb, prec, view=view, lower_only=lower, which=which)
    for gi, gj in [(70, 3), (200, 130), (383, 320), (5, 0)]:
        if not lower or gi >= gj:
            mat.A[gi, gj] += 7.0
    mat.colchk[2 * 3, 200] += 50.0
    tol = lib.abft_tol_t(ck.TOL_MAGNITUDE, 1.0, 0)
    r1, r2 = lib.Report.alloc(mat, deltas=True), lib.Report.alloc(mat, deltas=True)
    lib.abft_verify(mat, t, which, tol, r1)
    lib.abft_verify_gemm(mat, t, which, tol, r2)
    torch.cuda.synchronize()
    assert torch.equal(r1.status, r2.status) and torch.equal(r1.counts, r2.counts), (r1.counts, r2.counts)
    assert int(r1.counts[0]) >= 3
    # and both against the oracle's verify of the same corrupted state
    st = gpu_state_to_oracle(mat, prec)
    ost, ocnt = ck.verify(st, ck.Tiles(0, st.mt, 0, st.nt, lower, view), which)
    s2 = host(r2.status).astype(int)
    for (I, J), s in ost.items():
        assert s2[I, J] == s, ((I, J), s2[I, J], s)
    assert list(r2.counts.cpu().numpy()[:4]) == ocnt
    scale = {"f64": 1e-12, "f32": 1e-5}[prec] * float(mat.A.abs().sum(0).max())
    assert float((r1.dcol - r2.dcol).abs().max()) <= scale * nb
    if which & ck.ROW:
        assert float((r1.drow - r2.drow).abs().max()) <= scale * nb


def test_potrf_with_gemm_checks(lib):
    """ft_potrf with the checks' recalculation done by GEMMs (the paper's
    'without the optimized kernel' variant, L653): error free it equals LAPACK;
    a MUST-band fault is fixed exactly as with the fused pass."""
    ctx = lib.Context()
    A_np = si.spd(1024, seed=13)
    Lref = np.linalg.cholesky(A_np)
    inj = [(3, lib.AT_POST_TMU, lib.KIND_PERSIST, 0, 900, 700, 1 << 60),
           (2, lib.AT_PRE_PU_CHECK, lib.KIND_PERSIST, 0, 600, 300, 1 << 58)]
    outs = []
    for gemm in (False, True):
        for plan in ((), inj):
            A = dev(A_np)
            log = torch.zeros(1024 * lib.FIX_BYTES, dtype=torch.uint8, device="cuda")
            rc, info, st = lib.ft_potrf(ctx, A, 128, inject=plan, fix_log=log, checksum_gemm=gemm)
            torch.cuda.synchronize()
            L = np.tril(host(A))
            assert rc == 0 and info == 0
            assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()
            outs.append(sorted((f[0], f[1], f[4]) for f in lib.decode_fixes(log, st.n_fixes)))
    assert outs[0] == outs[2] == [] and outs[1] == outs[3] and len(outs[1]) == 2
