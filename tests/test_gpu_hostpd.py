"""GPU parity of the FT_PD_HOST drivers (Alg. 2 lines 3-7 with the PD on the
host, L364-L372; reading c-28) against the oracle drivers' pd_location="host"
mode and LAPACK, through the C ABI: fault-free factors, and D2H / H2D
transfer faults whose outcomes (host fixes, re-transfers, device fixes with
their positions and classes) must match the oracle's exactly."""
import numpy as np
import pytest
import scipy.linalg as sla
import torch

import synth_inputs as si
from oracle import drivers as dr
from tests.gpu_helpers import dev, host

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx(lib):
    c = lib.Context()
    c.set_host_lapack()
    return c


def _inj(k, point, gi, gj, bits=(62,), kind=dr.KIND_PERSIST):
    return dr.Inject(k, point, kind, 0, gi, gj, tuple(bits))


def _c(inject):
    return [(f.iter, f.point, f.kind, f.target, f.gi, f.gj, si.mask_of(f.bits)) for f in inject]


def _xfer(stats):
    return (stats.xfer_d2h_flagged, stats.xfer_d2h_fixed, stats.xfer_retransfers, stats.xfer_h2d_flagged,
            stats.xfer_h2d_fixed, stats.xfer_resends, stats.xfer_uncorrectable)


def _oxfer(st):
    x = st.xfer
    return (x.d2h_flagged, x.d2h_fixed, x.retransfers, x.h2d_flagged, x.h2d_fixed, x.resends, x.uncorrectable)


def _log(lib):
    return torch.zeros(8192 * lib.FIX_BYTES, dtype=torch.uint8, device="cuda")


def _run(lib, ctx, which, A_np, nb, inject=(), abft=True, pd=None):
    pd = lib.PD_HOST if pd is None else pd
    A = dev(A_np)
    n = A.shape[0]
    log = _log(lib)
    if which == "potrf":
        rc, info, stats = lib.ft_potrf(ctx, A, nb, abft=abft, inject=_c(inject), fix_log=log, pd_location=pd)
        extra = None
    elif which == "getrf":
        ipiv = torch.zeros(n, dtype=torch.int64, device="cuda")
        rc, info, stats = lib.ft_getrf(ctx, A, nb, ipiv, abft=abft, inject=_c(inject), fix_log=log, pd_location=pd)
        extra = ipiv
    else:
        tau = torch.zeros(n, dtype=torch.float64, device="cuda")
        rc, info, stats = lib.ft_geqrf(ctx, A, nb, tau, abft=abft, inject=_c(inject), fix_log=log, pd_location=pd)
        extra = tau
    torch.cuda.synchronize()
    out = host(A)
    if which == "potrf":
        out = np.tril(out)
    ex = None if extra is None else extra.cpu().numpy()
    return out, ex, rc, info, stats, lib.decode_fixes(log, stats.n_fixes)


@pytest.mark.parametrize("which", ["potrf", "getrf", "geqrf"])
@pytest.mark.parametrize("abft", [True, False])
def test_host_pd_fault_free_matches_lapack(lib, ctx, which, abft):
    n, nb = 1024, 128
    if which == "potrf":
        A = si.spd(n, seed=21)
        out, _, rc, info, stats, fixes = _run(lib, ctx, which, A, nb, abft=abft)
        ref = np.linalg.cholesky(A)
    elif which == "getrf":
        A = si.general(n, seed=22)
        out, piv, rc, info, stats, fixes = _run(lib, ctx, which, A, nb, abft=abft)
        ref, p = sla.lu_factor(A)
        assert np.array_equal(piv - 1, p)
    else:
        A = si.general(n, seed=23)
        out, tau, rc, info, stats, fixes = _run(lib, ctx, which, A, nb, abft=abft)
        h, t = np.linalg.qr(A, mode="raw")
        ref = h.T
        assert np.abs(tau - t).max() <= 1e-12
    assert rc == 0 and info == 0 and list(stats.counts) == [0] * 8 and not fixes
    assert _xfer(stats) == (0,) * 7
    assert np.abs(out - ref).max() <= 1e-12 * np.abs(ref).max()
    assert stats.ms_host_pd > 0


def _parity(lib, ctx, which, A, nb, inject):
    g_out, g_ex, rc, info, stats, gfix = _run(lib, ctx, which, A, nb, inject)
    if which == "potrf":
        o_out, ost = dr.ft_potrf(A, nb, inject=inject, pd_location="host", lookahead=True)
        ref, _ = dr.ft_potrf(A, nb)
    elif which == "getrf":
        o_out, o_piv, ost = dr.ft_getrf(A, nb, inject=inject, pd_location="host", lookahead=True)
        ref, _, _ = dr.ft_getrf(A, nb)
        assert np.array_equal(g_ex - 1, o_piv)
    else:
        o_out, o_tau, ost = dr.ft_geqrf(A, nb, inject=inject, pd_location="host")
        ref, _, _ = dr.ft_geqrf(A, nb)
        assert np.abs(g_ex - o_tau).max() <= 1e-12
    assert _xfer(stats) == _oxfer(ost)
    assert sorted((f[0], f[1], f[4]) for f in gfix) == sorted((f.gi, f.gj, f.cls) for f in ost.fixes)
    assert list(stats.counts) == ost.counts
    assert (rc == 0) == (ost.uncorrectable == 0)
    assert np.abs(g_out - o_out).max() <= 1e-12 * np.abs(o_out).max()
    return g_out, ref, stats


def test_potrf_transfer_faults_match_oracle(lib, ctx):
    n, nb = 512, 64
    A = si.spd(n, seed=24)
    inj = [_inj(1, dr.AT_D2H, nb + 5, nb + 3),
           _inj(3, dr.AT_H2D, 3 * nb + 9, 3 * nb + 1),
           _inj(5, dr.AT_D2H, 5 * nb + 1, 5 * nb + 0),
           _inj(5, dr.AT_D2H, 5 * nb + 7, 5 * nb + 0, (61,)),
           _inj(6, dr.AT_D2H, 6 * nb + 20, 6 * nb + 2, (52, 55))]
    out, ref, stats = _parity(lib, ctx, "potrf", A, nb, inj)
    assert np.abs(out - ref).max() <= 1e-12 * np.abs(ref).max()
    assert stats.xfer_retransfers == 1 and stats.xfer_h2d_fixed == 1 and stats.xfer_d2h_fixed == 2


def test_getrf_transfer_faults_match_oracle(lib, ctx):
    n, nb = 512, 64
    A = si.general(n, seed=25)
    inj = [_inj(0, dr.AT_D2H, 300, 7), _inj(2, dr.AT_H2D, 2 * nb + 40, 2 * nb + 3),
           _inj(4, dr.AT_H2D, 500, 4 * nb + 60, (60,))]
    out, ref, stats = _parity(lib, ctx, "getrf", A, nb, inj)
    assert np.abs(out - ref).max() <= 1e-12 * np.abs(ref).max()
    assert stats.xfer_h2d_fixed == 2 and stats.xfer_d2h_fixed == 1


def test_geqrf_transfer_faults_match_oracle(lib, ctx):
    n, nb = 512, 64
    A = si.general(n, seed=26)
    inj = [_inj(1, dr.AT_D2H, 100, nb + 5), _inj(3, dr.AT_H2D, 3 * nb + 3, 3 * nb + 60)]
    out, ref, stats = _parity(lib, ctx, "geqrf", A, nb, inj)
    assert np.abs(out - ref).max() <= 1e-12 * np.abs(ref).max()


def test_unprotected_transfer_fault_is_silent(lib, ctx):
    A = si.spd(256, seed=27)
    out, _, rc, info, stats, _ = _run(lib, ctx, "potrf", A, 32, [_inj(1, dr.AT_D2H, 40, 33, (52,))], abft=False)
    assert rc == 0 and not np.abs(out - np.linalg.cholesky(A)).max() <= 1e-6


def test_host_pd_needs_a_host_lapack(lib):
    bare = lib.Context()
    A = dev(si.spd(128, seed=1))
    with pytest.raises(lib.AbftError):
        lib.ft_potrf(bare, A, 32, pd_location=lib.PD_HOST)
