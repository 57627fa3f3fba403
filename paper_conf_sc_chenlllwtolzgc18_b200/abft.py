"""Thin ctypes binding of include/abft.h (argument marshalling only).

Every function here has the C name it forwards to; all arithmetic happens in
libabft_b200.so (sm_100a kernels + cuBLAS/cuSOLVER).  torch is used only to
allocate device memory and to name the current CUDA stream.  There is no CPU
fallback: if the library or a GPU is missing, loading fails loudly.

Layout: the C ABI is column-major.  A column-major m x n torch view is a
tensor of shape (m, n) with stride (1, ld); `colmajor_empty`/`to_colmajor`
make them.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import torch

from . import _lib

# ---------------------------------------------------------------- enums ----
F32, F64 = 0, 1
GENERAL, LOWER, UNIT_LOWER, UPPER, SYM_LOWER = 0, 1, 2, 3, 4
COL, ROW, BOTH = 1, 2, 3
TOL_MAGNITUDE, TOL_POSTERIORI = 0, 1
ST_COL, ST_ROW, ST_NONFINITE, ST_UNCORRECTABLE = 1, 2, 4, 8
CLS_CLEAN, CLS_0D, CLS_1D_ROW, CLS_1D_COL, CLS_SYM_CROSS = 0, 1, 2, 3, 4
CLS_CHK_CORRUPT, CLS_STALE_R, CLS_STALE_C, CLS_2D = 5, 6, 7, 8
FIX_DATA, FIX_COLCHK, FIX_ROWCHK = 0, 1, 2
NCOUNTS = 8
E_UNCORRECTABLE = 5
AT_PRE_PD_CHECK, AT_PRE_PD, AT_POST_PD, AT_PRE_PU_CHECK = 0, 1, 2, 3
AT_PRE_PU, AT_POST_PU, AT_PRE_TMU, AT_POST_TMU = 4, 5, 6, 7
AT_D2H, AT_H2D = 8, 9
KIND_PERSIST, KIND_ONCHIP = 0, 1
PD_DEVICE, PD_HOST = 0, 1
SCHEME_NEW, SCHEME_FULL_POST, SCHEME_SINGLE_POST, SCHEME_SINGLE_PRE = 0, 1, 2, 3  # ft_opts_t.scheme (c-34)


# ------------------------------------------------------------- structs ----
class abft_mat_t(C.Structure):
    _fields_ = [
        ("dtype", C.c_int32), ("m", C.c_int64), ("n", C.c_int64), ("nb", C.c_int64),
        ("A", C.c_void_p), ("lda", C.c_int64),
        ("colchk", C.c_void_p), ("ldc", C.c_int64),
        ("rowchk", C.c_void_p), ("ldr", C.c_int64),
        ("colmag", C.c_void_p), ("ldcm", C.c_int64),
        ("rowmag", C.c_void_p), ("ldrm", C.c_int64),
    ]


class abft_tiles_t(C.Structure):
    _fields_ = [("I0", C.c_int32), ("I1", C.c_int32), ("J0", C.c_int32), ("J1", C.c_int32),
                ("lower_only", C.c_int32), ("diag_view", C.c_int32)]


class abft_tol_t(C.Structure):
    _fields_ = [("kind", C.c_int32), ("scale", C.c_double), ("refresh", C.c_int32)]


class abft_report_t(C.Structure):
    _fields_ = [("status", C.c_void_p), ("ld_status", C.c_int64), ("dcol", C.c_void_p),
                ("drow", C.c_void_p), ("counts", C.c_void_p)]


class abft_fix_t(C.Structure):
    _fields_ = [("gi", C.c_int64), ("gj", C.c_int64), ("before", C.c_double), ("after", C.c_double),
                ("cls", C.c_int32), ("kind", C.c_int32)]


FIX_BYTES = C.sizeof(abft_fix_t)


class ft_inject_t(C.Structure):
    _fields_ = [("iter", C.c_int32), ("point", C.c_int32), ("kind", C.c_int32), ("target", C.c_int32),
                ("gi", C.c_int64), ("gj", C.c_int64), ("xor_mask", C.c_uint64)]


class ft_opts_t(C.Structure):
    _fields_ = [("nb", C.c_int64), ("abft", C.c_int32), ("tol_kind", C.c_int32), ("tol_scale", C.c_double),
                ("fig4a_repair", C.c_int32), ("n_inject", C.c_int32), ("inject", C.POINTER(ft_inject_t)),
                ("fix_log", C.c_void_p), ("fix_log_cap", C.c_int32), ("pu_gemm", C.c_int32),
                ("refresh", C.c_int32), ("restart", C.c_int32), ("pd_location", C.c_int32),
                ("fig4b", C.c_int32), ("trailing_check_period", C.c_int32), ("checksum_gemm", C.c_int32),
                ("scheme", C.c_int32), ("timing", C.c_int32), ("lookahead", C.c_int32)]


class ft_stats_t(C.Structure):
    _fields_ = [("counts", C.c_int32 * NCOUNTS), ("n_fixes", C.c_int32), ("repairs_applied", C.c_int32),
                ("repairs_skipped", C.c_int32), ("uncorrectable", C.c_int32), ("n_checks", C.c_int32),
                ("ms_total", C.c_double), ("restarts", C.c_int32),
                ("xfer_d2h_flagged", C.c_int32), ("xfer_d2h_fixed", C.c_int32), ("xfer_retransfers", C.c_int32),
                ("xfer_h2d_flagged", C.c_int32), ("xfer_h2d_fixed", C.c_int32), ("xfer_resends", C.c_int32),
                ("xfer_uncorrectable", C.c_int32), ("ms_host_pd", C.c_double),
                ("ctf_flagged", C.c_int32), ("ctf_recomputed", C.c_int32),
                ("detected", C.c_int32), ("corrected_0d", C.c_int32), ("corrected_1d", C.c_int32),
                ("checksum_repaired", C.c_int32), ("comm_errors", C.c_int32), ("ms_phase", C.c_double * 8)]


PHASES = ("pd", "pu", "tmu", "rules", "checks", "restart", "encode", "other")  # ft_stats_t.ms_phase


_L = _lib.load()
_vp, _i32, _i64, _u64, _d, _ch = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64, C.c_double, C.c_char
_P = C.POINTER
_sig = {
    "abft_encode": [_P(abft_mat_t), _P(abft_tiles_t), _i32, _vp],
    "abft_verify": [_P(abft_mat_t), _P(abft_tiles_t), _i32, _P(abft_tol_t), _P(abft_report_t), _vp],
    "abft_verify_gemm": [_P(abft_mat_t), _P(abft_tiles_t), _i32, _P(abft_tol_t), _P(abft_report_t), _vp],
    "abft_locate_correct": [_P(abft_mat_t), _P(abft_tiles_t), _i32, _P(abft_tol_t), _P(abft_report_t),
                            _vp, _i32, _vp, _vp],
    "abft_check": [_P(abft_mat_t), _P(abft_tiles_t), _i32, _P(abft_tol_t), _P(abft_report_t),
                   _vp, _i32, _vp, _vp],
    "abft_inject": [_vp, _i32, _i64, _u64, _vp],
    "abft_sizes": [_i64, _i64, _i64, _P(_i64), _P(_i64), _P(_i64), _P(_i64)],
    "abft_update_trsm": [_i32, _ch, _ch, _ch, _ch, _i64, _vp, _i64, _vp, _i64, _i64, _vp, _i64, _i64, _vp],
    "abft_update_gemm": [_i32, _i32, _ch, _ch, _d, _vp, _i64, _vp, _i64, _vp, _i64, _i64, _i64, _i64,
                         _vp, _i64, _vp, _i64, _vp],
    "abft_panel_potrf": [_P(abft_mat_t), _vp, _i64, _vp, _vp],
    "abft_tri_inverse": [_i32, _ch, _ch, _i64, _vp, _i64, _vp, _i64, _vp],
    "abft_update_trsm_inv": [_i32, _ch, _ch, _i64, _vp, _i64, _vp, _i64, _i64, _vp, _i64, _i64, _vp],
    "abft_update_syrk": [_i32, _i64, _i64, _vp, _i64, _vp, _i64, _vp, _i64, _vp, _vp, _i64, _vp, _vp, _i64, _vp],
    "abft_panel_getrf": [_P(abft_mat_t), _i32, _vp, _P(abft_tol_t), _P(abft_report_t), _vp, _i32, _vp, _vp, _vp,
                         _vp, _vp],
    "ft_getrf": [_vp, _i32, _i64, _vp, _i64, _vp, _P(ft_opts_t), _P(ft_stats_t), _P(_i64)],
    "abft_panel_geqrf": [_P(abft_mat_t), _i32, _vp, _vp, _vp, _vp, _vp, _vp],
    "ft_geqrf": [_vp, _i32, _i64, _vp, _i64, _vp, _P(ft_opts_t), _P(ft_stats_t), _P(_i64)],
    "ft_ctx_create": [_P(_vp), _i32, _vp],
    "ft_ctx_destroy": [_vp],
    "ft_potrf": [_vp, _i32, _i64, _vp, _i64, _P(ft_opts_t), _P(ft_stats_t), _P(_i64)],
    "ft_ctx_set_host_lapack": [_vp, C.c_char_p],
}
for _name, _args in _sig.items():
    _f = getattr(_L, _name)
    _f.argtypes = _args
    _f.restype = C.c_int32
EXPORTS = tuple(_sig)


class AbftError(RuntimeError):
    def __init__(self, name, rc):
        super().__init__(f"{name} returned {rc}")
        self.rc = rc


def _check(name, rc, ok=(0,)):
    if rc not in ok:
        raise AbftError(name, rc)
    return rc


# --------------------------------------------------------------- helpers ----
def _stream(stream):
    if stream is None:
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


def _dt(t: torch.Tensor) -> int:
    if t.dtype == torch.float64:
        return F64
    if t.dtype == torch.float32:
        return F32
    raise TypeError(f"unsupported dtype {t.dtype}")


def colmajor_empty(m, n, dtype=torch.float64, device="cuda", ld=None):
    ld = m if ld is None else ld
    buf = torch.empty((max(n, 1), max(ld, 1)), dtype=dtype, device=device)
    return buf[:n, :m].t()


def colmajor_zeros(m, n, dtype=torch.float64, device="cuda", ld=None):
    t = colmajor_empty(m, n, dtype, device, ld)
    t.zero_()
    return t


def to_colmajor(t: torch.Tensor, ld=None) -> torch.Tensor:
    m, n = t.shape
    out = colmajor_empty(m, n, t.dtype, t.device, ld)
    out.copy_(t)
    return out


def ld_of(t: torch.Tensor) -> int:
    """Leading dimension of a column-major 2-D view (stride (1, ld))."""
    if t is None:
        return 0
    m, n = t.shape
    if n > 1 and m > 1 and t.stride(0) != 1:
        raise ValueError("expected a column-major view (stride (1, ld))")
    return t.stride(1) if n > 1 else max(m, 1)


def _ptr(t):
    return None if t is None else t.data_ptr()


@dataclass
class Mat:
    """A matrix and its maintained checksum state (abft_mat_t)."""

    A: torch.Tensor
    nb: int
    colchk: torch.Tensor = None
    rowchk: torch.Tensor = None
    colmag: torch.Tensor = None
    rowmag: torch.Tensor = None

    @classmethod
    def alloc(cls, A: torch.Tensor, nb: int, mags: bool = True):
        m, n = A.shape
        mt, nt = m // nb, n // nb
        kw = dict(dtype=A.dtype, device=A.device)
        st = cls(A, nb, colmajor_zeros(2 * mt, n, **kw), colmajor_zeros(m, 2 * nt, **kw))
        if mags:
            st.colmag = colmajor_zeros(mt, n, **kw)
            st.rowmag = colmajor_zeros(m, nt, **kw)
        return st

    @property
    def mt(self):
        return self.A.shape[0] // self.nb

    @property
    def nt(self):
        return self.A.shape[1] // self.nb

    def c(self):
        m, n = self.A.shape
        return abft_mat_t(_dt(self.A), m, n, self.nb, _ptr(self.A), ld_of(self.A),
                          _ptr(self.colchk), ld_of(self.colchk), _ptr(self.rowchk), ld_of(self.rowchk),
                          _ptr(self.colmag), ld_of(self.colmag), _ptr(self.rowmag), ld_of(self.rowmag))


def tiles(I0, I1, J0, J1, lower_only=False, diag_view=GENERAL):
    return abft_tiles_t(I0, I1, J0, J1, int(lower_only), diag_view)


@dataclass
class Report:
    status: torch.Tensor  # int32 (mt x nt) column-major
    counts: torch.Tensor  # int32[8]
    dcol: torch.Tensor = None
    drow: torch.Tensor = None

    @classmethod
    def alloc(cls, mat: Mat, deltas=False):
        dev = mat.A.device
        st = colmajor_zeros(mat.mt, mat.nt, dtype=torch.int32, device=dev)
        cnt = torch.zeros(NCOUNTS, dtype=torch.int32, device=dev)
        r = cls(st, cnt)
        if deltas:
            r.dcol = torch.zeros_like(mat.colchk)
            r.drow = torch.zeros_like(mat.rowchk)
        return r

    def c(self):
        return abft_report_t(_ptr(self.status), ld_of(self.status), _ptr(self.dcol), _ptr(self.drow),
                             _ptr(self.counts))


# ------------------------------------------------------------ the C ABI ----
def abft_encode(mat: Mat, t: abft_tiles_t, which=BOTH, stream=None):
    m = mat.c()
    return _check("abft_encode", _L.abft_encode(C.byref(m), C.byref(t), which, _stream(stream)))


def abft_verify(mat: Mat, t: abft_tiles_t, which, tol: abft_tol_t, rep: Report, stream=None):
    m, r = mat.c(), rep.c()
    return _check("abft_verify", _L.abft_verify(C.byref(m), C.byref(t), which, C.byref(tol), C.byref(r),
                                                _stream(stream)))


def abft_verify_gemm(mat: Mat, t: abft_tiles_t, which, tol: abft_tol_t, rep: Report, stream=None):
    """Prior-art baseline: abft_verify with the checksums recomputed by cuBLAS GEMMs."""
    m, r = mat.c(), rep.c()
    return _check("abft_verify_gemm", _L.abft_verify_gemm(C.byref(m), C.byref(t), which, C.byref(tol), C.byref(r),
                                                          _stream(stream)))


def abft_locate_correct(mat: Mat, t: abft_tiles_t, which, tol: abft_tol_t, rep: Report,
                        fixes: torch.Tensor, n_fixes: torch.Tensor, stream=None):
    """fixes: uint8 device buffer of k*FIX_BYTES bytes; n_fixes: int32[1]."""
    m, r = mat.c(), rep.c()
    cap = 0 if fixes is None else fixes.numel() // FIX_BYTES
    return _check("abft_locate_correct",
                  _L.abft_locate_correct(C.byref(m), C.byref(t), which, C.byref(tol), C.byref(r), _ptr(fixes),
                                         cap, _ptr(n_fixes), _stream(stream)))


def abft_check(mat: Mat, t: abft_tiles_t, which, tol: abft_tol_t, rep: Report,
               fixes: torch.Tensor, n_fixes: torch.Tensor, stream=None):
    """abft_verify + abft_locate_correct in one launch (same arguments)."""
    m, r = mat.c(), rep.c()
    cap = 0 if fixes is None else fixes.numel() // FIX_BYTES
    return _check("abft_check",
                  _L.abft_check(C.byref(m), C.byref(t), which, C.byref(tol), C.byref(r), _ptr(fixes),
                                cap, _ptr(n_fixes), _stream(stream)))


def abft_inject(t: torch.Tensor, i: int, j: int, mask: int, stream=None):
    """XOR-flip element (i, j) of a column-major view."""
    off = i + j * ld_of(t)
    return _check("abft_inject", _L.abft_inject(_ptr(t), _dt(t), off, C.c_uint64(mask), _stream(stream)))


def abft_sizes(m, n, nb):
    out = [C.c_int64() for _ in range(4)]
    _check("abft_sizes", _L.abft_sizes(m, n, nb, *[C.byref(o) for o in out]))
    return tuple(o.value for o in out)


def abft_update_trsm(side, uplo, trans, diag, nb, T, chk, nvec, mag=None, nmag=0, stream=None):
    return _check("abft_update_trsm", _L.abft_update_trsm(
        _dt(T), side.encode(), uplo.encode(), trans.encode(), diag.encode(), nb, _ptr(T), ld_of(T),
        _ptr(chk), ld_of(chk), nvec, _ptr(mag), ld_of(mag), nmag, _stream(stream)))


def abft_update_gemm(which, transX, transY, alpha, Xchk, Y, Cchk, M2, N, K, Xmag=None, Cmag=None, stream=None):
    return _check("abft_update_gemm", _L.abft_update_gemm(
        _dt(Y), which, transX.encode(), transY.encode(), float(alpha), _ptr(Xchk), ld_of(Xchk), _ptr(Y), ld_of(Y),
        _ptr(Cchk), ld_of(Cchk), M2, N, K, _ptr(Xmag), ld_of(Xmag), _ptr(Cmag), ld_of(Cmag), _stream(stream)))


def abft_panel_potrf(diag: Mat, info: torch.Tensor, Linv: torch.Tensor = None, stream=None):
    m = diag.c()
    return _check("abft_panel_potrf", _L.abft_panel_potrf(C.byref(m), _ptr(Linv), ld_of(Linv) if Linv is not None
                                                          else 0, _ptr(info), _stream(stream)))


def abft_tri_inverse(uplo, diag, T, W, stream=None):
    nb = T.shape[0]
    return _check("abft_tri_inverse", _L.abft_tri_inverse(_dt(T), uplo.encode(), diag.encode(), nb, _ptr(T), ld_of(T),
                                                          _ptr(W), ld_of(W), _stream(stream)))


def abft_update_trsm_inv(side, trans, W, chk, nvec, mag=None, nmag=0, stream=None):
    return _check("abft_update_trsm_inv", _L.abft_update_trsm_inv(
        _dt(W), side.encode(), trans.encode(), W.shape[0], _ptr(W), ld_of(W), _ptr(chk), ld_of(chk), nvec,
        _ptr(mag), ld_of(mag), nmag, _stream(stream)))


def abft_update_syrk(nb, ntk, L21, cL, Cc, Rr, mL=None, Cm=None, Rm=None, stream=None):
    """Cholesky TMU checksum rule; Cc/Rr/Cm/Rm are the trailing blocks of
    colchk/rowchk/colmag/rowmag (views sharing their arrays' ld)."""
    return _check("abft_update_syrk", _L.abft_update_syrk(
        _dt(L21), nb, ntk, _ptr(L21), ld_of(L21), _ptr(cL), ld_of(cL), _ptr(mL), ld_of(mL), _ptr(Cc), _ptr(Rr),
        ld_of(Rr), _ptr(Cm), _ptr(Rm), ld_of(Rm), _stream(stream)))


def decode_fixes(buf: torch.Tensor, n: int):
    """Device fix records -> list of (gi, gj, before, after, cls, kind)."""
    n = min(n, buf.numel() // FIX_BYTES)
    raw = bytes(buf[: n * FIX_BYTES].cpu().numpy().tobytes())
    arr = (abft_fix_t * n).from_buffer_copy(raw)
    return [(f.gi, f.gj, f.before, f.after, f.cls, f.kind) for f in arr]


class Context:
    """ft_ctx_t owner (cuBLAS/cuSOLVER handles are per device inside the lib)."""

    def __init__(self, device=None, stream=None):
        dev = torch.cuda.current_device() if device is None else device
        self._h = C.c_void_p()
        _check("ft_ctx_create", _L.ft_ctx_create(C.byref(self._h), dev, _stream(stream)))

    def set_host_lapack(self, path=None):
        """Host LAPACK for pd_location=PD_HOST (Alg. 2's CPU panel, L61):
        `path` to a shared library with LP64 dpotrf_/dgetrf_/dgeqrf_ (and the
        s-variants); default: the OpenBLAS bundled with SciPy."""
        if path is None:
            path = host_lapack_path()
        _check("ft_ctx_set_host_lapack", _L.ft_ctx_set_host_lapack(self._h, path.encode()))
        self.host_lapack = path

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and _L is not None:
            _L.ft_ctx_destroy(h)
            self._h = None


def host_lapack_path():
    """The LP64 OpenBLAS shipped in scipy.libs (exports scipy_dpotrf_ etc.)."""
    import glob

    import scipy

    libs = os.path.join(os.path.dirname(os.path.dirname(scipy.__file__)), "scipy.libs")
    cands = sorted(glob.glob(os.path.join(libs, "libscipy_openblas-*.so")))
    if not cands:
        raise FileNotFoundError(f"no libscipy_openblas-*.so under {libs}")
    return cands[0]


def _opts(nb, abft, tol_kind, tol_scale, fig4a_repair, inject, fix_log, pu_gemm, refresh=True, restart=True,
          pd_location=PD_DEVICE, fig4b=True, period=0, scheme=0, checksum_gemm=False, lookahead=False,
          timing=False):
    inj = (ft_inject_t * max(1, len(inject)))()
    for k, f in enumerate(inject):
        inj[k] = ft_inject_t(*f)
    opts = ft_opts_t(nb, int(abft), tol_kind, tol_scale, int(fig4a_repair), len(inject), inj,
                     _ptr(fix_log), 0 if fix_log is None else fix_log.numel() // FIX_BYTES, int(pu_gemm),
                     int(refresh), int(restart), int(pd_location), int(fig4b), int(period), int(checksum_gemm),
                     int(scheme), int(timing), int(lookahead))
    return opts, inj


def abft_panel_getrf(mat: Mat, k: int, ipiv: torch.Tensor, Linv: torch.Tensor, Uinv: torch.Tensor,
                     info: torch.Tensor, tol: abft_tol_t = None, rep: Report = None, fixes: torch.Tensor = None,
                     n_fixes: torch.Tensor = None, stream=None):
    m = mat.c()
    r = rep.c() if rep is not None else None
    cap = 0 if fixes is None else fixes.numel() // FIX_BYTES
    return _check("abft_panel_getrf", _L.abft_panel_getrf(
        C.byref(m), k, _ptr(ipiv), C.byref(tol) if tol is not None else None, C.byref(r) if r is not None else None,
        _ptr(fixes), cap, _ptr(n_fixes), _ptr(Linv), _ptr(Uinv), _ptr(info), _stream(stream)))


def ft_getrf(ctx: Context, A: torch.Tensor, nb: int, ipiv: torch.Tensor, abft=True, tol_kind=TOL_MAGNITUDE,
             tol_scale=1.0, fig4a_repair=True, inject=(), fix_log=None, pd_location=PD_DEVICE, restart=True,
             fig4b=True, trailing_check_period=0, timing=False, lookahead=True):
    """Fault-tolerant LU with partial pivoting in place on a column-major A;
    ipiv: int64 device tensor (n), receives 1-based global pivots."""
    n = A.shape[0]
    opts, _inj = _opts(nb, abft, tol_kind, tol_scale, fig4a_repair, inject, fix_log, True, restart=restart,
                       pd_location=pd_location, fig4b=fig4b, period=trailing_check_period, timing=timing,
                       lookahead=lookahead)
    stats = ft_stats_t()
    info = C.c_int64()
    rc = _L.ft_getrf(ctx._h, _dt(A), n, _ptr(A), ld_of(A), _ptr(ipiv), C.byref(opts), C.byref(stats),
                     C.byref(info))
    _check("ft_getrf", rc, ok=(0, E_UNCORRECTABLE))
    return rc, info.value, stats


def abft_panel_geqrf(mat: Mat, k: int, tau: torch.Tensor, V: torch.Tensor, T: torch.Tensor,
                     panel_copy: torch.Tensor, info: torch.Tensor, stream=None):
    m = mat.c()
    return _check("abft_panel_geqrf", _L.abft_panel_geqrf(C.byref(m), k, _ptr(tau), _ptr(V), _ptr(T),
                                                          _ptr(panel_copy), _ptr(info), _stream(stream)))


def ft_geqrf(ctx: Context, A: torch.Tensor, nb: int, tau: torch.Tensor, abft=True, tol_kind=TOL_MAGNITUDE,
             tol_scale=1.0, inject=(), fix_log=None, pd_location=PD_DEVICE, restart=True, trailing_check_period=0,
             timing=False):
    """Fault-tolerant Householder QR in place on a column-major A (LAPACK
    dgeqrf storage); tau: device tensor (n) of A's dtype."""
    n = A.shape[0]
    opts, _inj = _opts(nb, abft, tol_kind, tol_scale, True, inject, fix_log, True, restart=restart,
                       pd_location=pd_location, period=trailing_check_period, timing=timing)
    stats = ft_stats_t()
    info = C.c_int64()
    rc = _L.ft_geqrf(ctx._h, _dt(A), n, _ptr(A), ld_of(A), _ptr(tau), C.byref(opts), C.byref(stats),
                     C.byref(info))
    _check("ft_geqrf", rc, ok=(0, E_UNCORRECTABLE))
    return rc, info.value, stats


def ft_potrf(ctx: Context, A: torch.Tensor, nb: int, abft=True, tol_kind=TOL_MAGNITUDE, tol_scale=1.0,
             fig4a_repair=True, inject=(), fix_log=None, pu_gemm=True, refresh=True, restart=True,
             pd_location=PD_DEVICE, fig4b=True, trailing_check_period=0, scheme=0, checksum_gemm=False,
             lookahead=True, timing=False):
    """Fault-tolerant lower Cholesky in place on a column-major A.  Returns
    (rc, info, stats) with rc 0 or E_UNCORRECTABLE (other codes raise).
    pd_location=PD_HOST needs ctx.set_host_lapack() first.  scheme: SCHEME_*
    (the checking scheme, include/abft.h ft_opts_t.scheme); checksum_gemm: the
    checks recompute checksums by GEMMs (prior-art baseline, abft_verify_gemm);
    lookahead: the next panel's PD / PU next to the TMU (reading c-35)."""
    n = A.shape[0]
    opts, _inj = _opts(nb, abft, tol_kind, tol_scale, fig4a_repair, inject, fix_log, pu_gemm, refresh, restart,
                       pd_location, fig4b, trailing_check_period, scheme, checksum_gemm, lookahead, timing)
    stats = ft_stats_t()
    info = C.c_int64()
    rc = _L.ft_potrf(ctx._h, _dt(A), n, _ptr(A), ld_of(A), C.byref(opts), C.byref(stats), C.byref(info))
    _check("ft_potrf", rc, ok=(0, E_UNCORRECTABLE))
    return rc, info.value, stats
