"""GPU parity of ft_potrf's checking schemes (ft_opts_t.scheme, reading c-34;
the schemes the paper compares, L542 Table VIII, L653 Figs. 12-14) against the
oracle driver through the C ABI: error-free factors, the number of checks,
and fault cases whose fix logs / outcomes must match the oracle's exactly."""
import numpy as np
import pytest
import torch

import synth_inputs as si
from oracle import drivers as dr
from tests.gpu_helpers import dev, host
from tests.test_oracle_drivers import SCHEME_OUTCOMES, SCHEMES

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx(lib):
    return lib.Context()


def _gpu(lib, ctx, A_np, nb, scheme, inject=()):
    A = dev(A_np)
    inj = [(f.iter, f.point, f.kind, f.target, f.gi, f.gj, si.mask_of(f.bits)) for f in inject]
    log = torch.zeros(8192 * lib.FIX_BYTES, dtype=torch.uint8, device="cuda")
    rc, info, stats = lib.ft_potrf(ctx, A, nb, inject=inj, fix_log=log, scheme=scheme)
    torch.cuda.synchronize()
    return np.tril(host(A)), rc, stats, lib.decode_fixes(log, stats.n_fixes)


@pytest.mark.parametrize("scheme", SCHEMES)
@pytest.mark.parametrize("n,nb", [(256, 32), (2048, 256)])
def test_scheme_error_free(lib, ctx, scheme, n, nb):
    A = si.spd(n, seed=n + scheme)
    L, rc, st, fixes = _gpu(lib, ctx, A, nb, scheme)
    _, so = dr.ft_potrf(A, nb, scheme=scheme, lookahead=True)
    Lref = np.linalg.cholesky(A)
    assert rc == 0 and list(st.counts) == [0] * 8 and not fixes
    assert st.n_checks == so.n_checks
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()


@pytest.mark.parametrize("scheme", SCHEMES)
@pytest.mark.parametrize("case", range(len(SCHEME_OUTCOMES)))
def test_scheme_fault_parity(lib, ctx, scheme, case):
    f, expect = SCHEME_OUTCOMES[case]
    A = si.spd(256, seed=3)
    Lo, so = dr.ft_potrf(A, 32, inject=[f], scheme=scheme, lookahead=True)
    Lg, rc, sg, fg = _gpu(lib, ctx, A, 32, scheme, inject=[f])
    assert (rc == lib.E_UNCORRECTABLE) == (so.uncorrectable > 0) == (expect[scheme] == "R")
    assert sg.restarts == so.restarts
    assert list(sg.counts) == so.counts, (list(sg.counts), so.counts)
    assert sorted((x[0], x[1], x[4], x[5]) for x in fg) == sorted((x.gi, x.gj, x.cls, x.kind) for x in so.fixes)
    if expect[scheme] == "Y":
        Lref = np.linalg.cholesky(A)
        assert np.abs(Lg - Lref).max() <= 1e-12 * np.abs(Lref).max()


def test_scheme_rejected_by_lu_qr(lib, ctx):
    A = dev(si.general(128, seed=1))
    ipiv = torch.zeros(128, dtype=torch.int64, device="cuda")
    opts, _inj = lib._opts(32, True, lib.TOL_MAGNITUDE, 1.0, True, (), None, True, scheme=lib.SCHEME_FULL_POST)
    stats = lib.ft_stats_t()
    import ctypes as C
    info = C.c_int64()
    rc = lib._L.ft_getrf(lib.Context()._h, lib._dt(A), 128, lib._ptr(A), lib.ld_of(A), lib._ptr(ipiv),
                         C.byref(opts), C.byref(stats), C.byref(info))
    assert rc == -7
