"""GPU parity of ft_getrf (LU rows of §8 a4–a7) against the oracle driver
and LAPACK (BASELINE configs[2] shape), through the C ABI."""
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
    return lib.Context()


def _gpu_getrf(lib, ctx, A_np, nb, inject=(), abft=True, fig4a=True, dtype=torch.float64, lookahead=True):
    A = dev(A_np, dtype)
    n = A.shape[0]
    ipiv = torch.zeros(n, dtype=torch.int64, device="cuda")
    inj = [(f.iter, f.point, f.kind, f.target, f.gi, f.gj, si.mask_of(f.bits)) for f in inject]
    log = torch.zeros(8192 * lib.FIX_BYTES, dtype=torch.uint8, device="cuda")
    rc, info, stats = lib.ft_getrf(ctx, A, nb, ipiv, abft=abft, fig4a_repair=fig4a, inject=inj, fix_log=log,
                                   lookahead=lookahead)
    torch.cuda.synchronize()
    return host(A), ipiv.cpu().numpy() - 1, rc, info, stats, lib.decode_fixes(log, stats.n_fixes)


@pytest.mark.parametrize("lookahead", [True, False])
@pytest.mark.parametrize("n,nb", [(256, 32), (1024, 128), (2048, 256), (2048, 512), (4096, 1024)])
def test_error_free_matches_lapack(lib, ctx, n, nb, lookahead):
    A = si.general(n, seed=n)
    LU, piv, rc, info, stats, fixes = _gpu_getrf(lib, ctx, A, nb, lookahead=lookahead)
    if n <= 1024:  # the check sequence of Alg. 2 (with the look-ahead's extra re-checks, c-35)
        assert stats.n_checks == dr.ft_getrf(A, nb, lookahead=lookahead)[2].n_checks
    lu, p = sla.lu_factor(A)
    assert rc == 0 and info == 0 and list(stats.counts) == [0] * 8 and not fixes
    assert np.array_equal(piv, p)
    if n <= 1024:
        assert np.abs(LU - lu).max() <= 1e-12 * np.abs(lu).max()
    else:
        # two different LU evaluation orders differ by ~cond(A)·u elementwise at
        # large n; compare backward errors instead: ||P A - L U|| <= 32 n u ||A||
        L = np.tril(LU, -1) + np.eye(n)
        U = np.triu(LU)
        PA = A.copy()
        for i, j in enumerate(piv):
            if j != i:
                PA[[i, j]] = PA[[j, i]]
        assert np.abs(PA - L @ U).max() <= 32 * n * 2.0 ** -53 * np.abs(A).max() * n ** 0.5


def test_unprotected_same_factor(lib, ctx):
    A = si.general(1024, seed=2)
    a = _gpu_getrf(lib, ctx, A, 128, abft=False)
    b = _gpu_getrf(lib, ctx, A, 128, abft=True)
    assert np.array_equal(a[1], b[1])
    assert np.abs(a[0] - b[0]).max() <= 1e-13 * np.abs(a[0]).max()


def _compare(lib, ctx, A, nb, injects, prec="f64", lookahead=True):
    """fp32: the GPU factors in fp32; the oracle carries the fp32 input, fp32
    flips and fp32 thresholds in fp64 arithmetic (pivots must still agree)."""
    vtol = 1e-12 if prec == "f64" else 1e-5
    if prec == "f32":
        A = A.astype(np.float32).astype(np.float64)
    LUo, pivo, so = dr.ft_getrf(A, nb, prec=prec, inject=injects, lookahead=lookahead)
    LUg, pivg, rc, info, sg, fg = _gpu_getrf(lib, ctx, A, nb, inject=injects,
                                             dtype=torch.float64 if prec == "f64" else torch.float32,
                                             lookahead=lookahead)
    assert (rc == lib.E_UNCORRECTABLE) == (so.uncorrectable > 0)
    assert sg.repairs_skipped == so.repairs_skipped
    if so.repairs_skipped:
        return so, sg
    # fp32: counts[3] (tiles with a non-finite delta) records fp32 overflow of
    # the recomputed sums, which the oracle (fp32 data summed in fp64) cannot see
    nf = [3] if prec == "f32" else []
    assert [c for i, c in enumerate(sg.counts) if i not in nf] == [c for i, c in enumerate(so.counts) if i not in nf], \
        (list(sg.counts), so.counts)
    assert sorted((f[0], f[1], f[4], f[5]) for f in fg) == sorted((f.gi, f.gj, f.cls, f.kind) for f in so.fixes)
    assert sg.repairs_applied == so.repairs_applied
    assert sg.n_checks == so.n_checks
    if so.uncorrectable == 0:
        lu, p = sla.lu_factor(A)
        assert np.array_equal(pivg, p) and np.array_equal(pivo, p)
        assert np.abs(LUg - lu).max() <= vtol * np.abs(lu).max()
    return so, sg


LU_CASES = [
    (2, dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 0, 100, 70, (61,)),
    (2, dr.AT_POST_PD, dr.KIND_PERSIST, 0, 150, 80, (62,)),
    (2, dr.AT_POST_PD, dr.KIND_PERSIST, 0, 66, 90, (58,)),
    (2, dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 0, 70, 200, (60,)),
    (2, dr.AT_POST_PU, dr.KIND_PERSIST, 0, 75, 180, (63,)),
    (2, dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 72, 130, (57,)),
    (2, dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 80, 70, (57,)),     # L_kk read by the PU -> 2D (R)
    (2, dr.AT_PRE_TMU, dr.KIND_ONCHIP, 0, 140, 72, (57,)),
    (2, dr.AT_PRE_TMU, dr.KIND_ONCHIP, 0, 70, 140, (56,)),
    (2, dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 170, 80, (54,)),
    (2, dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 80, 170, (55,)),
    (2, dr.AT_POST_TMU, dr.KIND_PERSIST, 0, 230, 100, (59,)),
    (1, dr.AT_POST_TMU, dr.KIND_PERSIST, 0, 70, 200, (60,)),  # moved by the next pivoting (c-14b)
    (2, dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 2, 70, 13, (60,)),  # row-checksum memory fault
    (2, dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 1, 9, 75, (61,)),   # column-checksum memory fault
]


@pytest.mark.parametrize("lookahead", [True, False])
@pytest.mark.parametrize("case", range(len(LU_CASES)))
def test_lu_fault_campaign_parity(lib, ctx, case, lookahead):
    k, point, kind, target, gi, gj, bits = LU_CASES[case]
    A = si.general(256, seed=0)
    _compare(lib, ctx, A, 32, [dr.Inject(k, point, kind, target, gi, gj, bits)], lookahead=lookahead)


@pytest.mark.parametrize("case", range(len(LU_CASES)))
def test_lu_fault_campaign_parity_f32(lib, ctx, case):
    """The same fault kinds in fp32 (fp64 bit b -> fp32 bit b - 32)."""
    k, point, kind, target, gi, gj, bits = LU_CASES[case]
    A = si.general(256, seed=0)
    _compare(lib, ctx, A, 32, [dr.Inject(k, point, kind, target, gi, gj, tuple(b - 32 for b in bits))], prec="f32")


def _random_lu_plan(n, nb, seed):
    g = si.rng(seed)
    nt = n // nb
    k = int(g.integers(0, nt - 1))
    point = int(g.integers(0, 8))
    kind = dr.KIND_ONCHIP if point in (dr.AT_PRE_PU, dr.AT_PRE_TMU) and g.random() < 0.5 else dr.KIND_PERSIST
    r0, r1 = k * nb, (k + 1) * nb
    if point in (dr.AT_PRE_PD_CHECK, dr.AT_PRE_PD, dr.AT_POST_PD):
        gi, gj = int(g.integers(r0, n)), int(g.integers(r0, r1))
    elif point in (dr.AT_PRE_PU_CHECK, dr.AT_PRE_PU, dr.AT_POST_PU):
        gi, gj = int(g.integers(r0, r1)), int(g.integers(r1, n))
    elif point == dr.AT_PRE_TMU:
        if g.random() < 0.5:
            gi, gj = int(g.integers(r1, n)), int(g.integers(r0, r1))
        else:
            gi, gj = int(g.integers(r0, r1)), int(g.integers(r1, n))
    else:
        gi, gj = int(g.integers(r1, n)), int(g.integers(r1, n))
    return [dr.Inject(k, point, kind, 0, gi, gj, (int(g.integers(52, 64)),))]


@pytest.mark.parametrize("seed", range(12))
def test_lu_random_campaign_parity(lib, ctx, seed):
    A = si.general(256, seed=200 + seed)
    _compare(lib, ctx, A, 32, _random_lu_plan(256, 32, seed))


def test_config3_shape_error_free(lib, ctx):
    """BASELINE configs[2]: fp64 LU n=20480 nb=512, error free; sampled rows
    of P·A − L·U against the input (a property that holds at any size)."""
    n, nb = 20480, 512
    A0 = si.general_device(n, seed=11)
    A = A0.clone()
    ipiv = torch.zeros(n, dtype=torch.int64, device="cuda")
    rc, info, stats = lib.ft_getrf(ctx, A, nb, ipiv)
    torch.cuda.synchronize()
    assert rc == 0 and info == 0 and list(stats.counts) == [0] * 8
    # apply the row interchanges to a copy of A0 (LAPACK order)
    perm = torch.arange(n, device="cuda")
    pv = (ipiv - 1).cpu().numpy()
    pm = perm.cpu().numpy()
    for i in range(n):
        j = pv[i]
        if j != i:
            pm[i], pm[j] = pm[j], pm[i]
    g = si.rng(3)
    rows = torch.tensor(sorted(g.choice(n, 32, replace=False)), device="cuda")
    L = torch.tril(A, -1)
    L.diagonal().fill_(1.0)
    U = torch.triu(A)
    PA = A0[torch.tensor(pm, device="cuda")[rows]]
    R = PA - L[rows] @ U
    assert R.abs().max().item() <= 1e-10 * A0.abs().max().item() * n ** 0.5


# ---- f1 local restart (L430): parity with the oracle's restart -------------
def _gpu_getrf_rs(lib, ctx, A_np, nb, inject, restart):
    A = dev(A_np)
    ipiv = torch.zeros(A.shape[0], dtype=torch.int64, device="cuda")
    inj = [(f.iter, f.point, f.kind, f.target, f.gi, f.gj, si.mask_of(f.bits)) for f in inject]
    rc, info, stats = lib.ft_getrf(ctx, A, nb, ipiv, inject=inj, restart=restart)
    torch.cuda.synchronize()
    return host(A), ipiv.cpu().numpy() - 1, rc, stats


# Two faults in one iteration: the first corrected by the pre-PD / pre-PU
# check, the second forcing the restart of that op.  The restart restores
# the input from the copy the check's own pass wrote (ft_driver.cuh
# check(ckpt)), which must hold the corrected element as the oracle's does.
LU_DOUBLE = [
    [(1, dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 0, 150, 70, (61,)), (1, dr.AT_PRE_PD, dr.KIND_PERSIST, 0, 130, 70, (60,))],
    [(2, dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 0, 130, 200, (60,)), (2, dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 140, 130, (60,))],
]


@pytest.mark.parametrize("lookahead", [True, False])
@pytest.mark.parametrize("case", range(len(LU_DOUBLE)))
def test_lu_restart_from_check_checkpoint(lib, ctx, case, lookahead):
    A = si.general(256, seed=31)
    so, sg = _compare(lib, ctx, A, 64, [dr.Inject(*c) for c in LU_DOUBLE[case]], lookahead=lookahead)
    assert so.restarts == 1 and sg.restarts == so.restarts


@pytest.mark.parametrize("k,point,kind,gi,gj,bit", [
    (1, dr.AT_PRE_PD, dr.KIND_PERSIST, 200, 66, 62),   # consumed by getrf, other pivots
    (1, dr.AT_PRE_PD, dr.KIND_PERSIST, 130, 70, 60),
    (1, dr.AT_PRE_PD, dr.KIND_PERSIST, 64, 64, 55),
    (2, dr.AT_PRE_PU, dr.KIND_ONCHIP, 140, 130, 60),   # L_kk read by the PU: U12 2D
])
def test_lu_restart_parity(lib, ctx, k, point, kind, gi, gj, bit):
    nb = 64
    A = si.general(256, seed=31)
    inj = [dr.Inject(k, point, kind, 0, gi, gj, (bit,))]
    ref, pref, _ = dr.ft_getrf(A, nb)
    o_lu, o_piv, ost = dr.ft_getrf(A, nb, inject=inj, lookahead=True)
    LU, piv, rc, st = _gpu_getrf_rs(lib, ctx, A, nb, inj, True)
    assert ost.restarts == 1 and ost.uncorrectable == 0
    assert rc == 0 and st.restarts == 1 and st.uncorrectable == 0
    assert list(st.counts) == ost.counts and st.n_checks == ost.n_checks
    assert np.array_equal(piv, pref)
    assert np.abs(LU - ref).max() <= 1e-12 * np.abs(ref).max()
    _, _, rc0, st0 = _gpu_getrf_rs(lib, ctx, A, nb, inj, False)
    assert rc0 == lib.E_UNCORRECTABLE and st0.restarts == 0
