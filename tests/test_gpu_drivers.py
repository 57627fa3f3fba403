"""GPU parity of ft_potrf (§8 rows a4–a7) against the oracle driver, through
the C ABI: error-free factors, and fault campaigns whose fix logs (positions,
classes) must match the oracle's exactly (BASELINE configs[0] and [1])."""
import numpy as np
import pytest
import torch

import synth_inputs as si
from oracle import checksum as ck
from oracle import drivers as dr
from tests.gpu_helpers import dev, host

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx(lib):
    return lib.Context()


def _gpu_potrf(lib, ctx, A_np, nb, inject=(), abft=True, fig4a=True, dtype=torch.float64, lookahead=True):
    A = dev(A_np, dtype)
    inj = [(f.iter, f.point, f.kind, f.target, f.gi, f.gj, si.mask_of(f.bits)) for f in inject]
    log = torch.zeros(8192 * lib.FIX_BYTES, dtype=torch.uint8, device="cuda")
    rc, info, stats = lib.ft_potrf(ctx, A, nb, abft=abft, fig4a_repair=fig4a, inject=inj, fix_log=log,
                                   lookahead=lookahead)
    torch.cuda.synchronize()
    fixes = lib.decode_fixes(log, stats.n_fixes)
    return np.tril(host(A)), rc, info, stats, fixes


@pytest.mark.parametrize("lookahead", [True, False])
@pytest.mark.parametrize("n,nb", [(256, 32), (1024, 128), (2048, 256), (2048, 512), (4096, 1024)])
def test_error_free_matches_lapack(lib, ctx, n, nb, lookahead):
    A = si.spd(n, seed=n)
    L, rc, info, stats, fixes = _gpu_potrf(lib, ctx, A, nb, lookahead=lookahead)
    Lref = np.linalg.cholesky(A)
    assert rc == 0 and info == 0 and stats.counts[:] == [0] * 8 and not fixes
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()
    # Alg. 2: 5 checks per iteration, 2 in the last; look-ahead adds the
    # panel re-check after the tile-column update (reading c-35)
    assert stats.n_checks == (6 if lookahead else 5) * (n // nb - 1) + 2


@pytest.mark.parametrize("lookahead", [True, False])
def test_unprotected_same_factor(lib, ctx, lookahead):
    A = si.spd(1024, seed=1)
    L0, *_ = _gpu_potrf(lib, ctx, A, 128, abft=False, lookahead=lookahead)
    L1, *_ = _gpu_potrf(lib, ctx, A, 128, abft=True, lookahead=lookahead)
    assert np.abs(L0 - L1).max() <= 1e-13 * np.abs(L0).max()


def test_not_spd_info(lib, ctx):
    A = si.spd(128, seed=4)
    A[70, 70] = -1e6
    _, rc, info, _, _ = _gpu_potrf(lib, ctx, A, 32, abft=False)
    assert info == 64 + 7


def _compare(lib, ctx, A, nb, injects, fig4a=True, prec="f64", lookahead=True):
    """Same fault plan on the oracle driver and the GPU driver: counters, fix
    positions / classes / kinds, restarts and repairs identical; factors
    within 1e-12 (fp64) / 1e-5 (fp32) of LAPACK's.  fp32: the GPU factors in
    fp32, the oracle carries fp32 inputs, fp32 flips and fp32 thresholds
    (u = 2^-24) in fp64 arithmetic; MUST-band faults take the same decisions."""
    vtol = 1e-12 if prec == "f64" else 1e-5
    if prec == "f32":
        A = A.astype(np.float32).astype(np.float64)
    Lo, so = dr.ft_potrf(A, nb, prec=prec, inject=injects, fig4a_repair=fig4a, lookahead=lookahead)
    Lg, rc, info, sg, fg = _gpu_potrf(lib, ctx, A, nb, inject=injects, fig4a=fig4a,
                                      dtype=torch.float64 if prec == "f64" else torch.float32, lookahead=lookahead)
    assert (rc == lib.E_UNCORRECTABLE) == (so.uncorrectable > 0)
    assert sg.repairs_skipped == so.repairs_skipped
    if so.repairs_skipped:
        # a guarded-out repair leaves overflowing garbage in the trailing
        # matrix: the outcome is R (detected, restart); what the checks see
        # afterwards is Inf/NaN arithmetic and not compared
        return so, sg
    assert sg.n_checks == so.n_checks
    # fp32: counts[3] (tiles with a non-finite delta) records fp32 overflow of
    # the recomputed sums, which the oracle (fp32 data summed in fp64) cannot see
    nf = [3] if prec == "f32" else []
    assert [c for i, c in enumerate(sg.counts) if i not in nf] == [c for i, c in enumerate(so.counts) if i not in nf], \
        (list(sg.counts), so.counts)
    assert sorted((f[0], f[1], f[4], f[5]) for f in fg) == sorted((f.gi, f.gj, f.cls, f.kind) for f in so.fixes)
    assert sg.repairs_applied == so.repairs_applied and sg.repairs_skipped == so.repairs_skipped
    assert sg.restarts == so.restarts
    assert (rc == lib.E_UNCORRECTABLE) == (so.uncorrectable > 0)
    if so.uncorrectable == 0:
        Lref = np.linalg.cholesky(A)
        assert np.abs(Lg - Lref).max() <= vtol * np.abs(Lref).max()
        assert np.abs(Lo - Lref).max() <= vtol * np.abs(Lref).max()
    return so, sg


# (point, kind, target, gi, gj, bits) at iteration 2, n=256, nb=32
CASES = [
    (dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 0, 70, 66, (61,)),
    (dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 0, 75, 75, (55, 52)),
    (dr.AT_POST_PD, dr.KIND_PERSIST, 0, 80, 70, (62,)),
    (dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 0, 200, 70, (60,)),
    (dr.AT_POST_PU, dr.KIND_PERSIST, 0, 150, 90, (63,)),
    (dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 130, 68, (58,)),
    (dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 70, 66, (60,)),      # PU reference part -> 2D -> local restart
    (dr.AT_PRE_PD, dr.KIND_PERSIST, 0, 70, 66, (57,)),     # consumed by the PD -> 2D -> local restart
    (dr.AT_PRE_TMU, dr.KIND_ONCHIP, 0, 140, 72, (57,)),
    (dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 170, 80, (54,)),    # Fig. 4a repair
    (dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 170, 80, (62,)),    # guarded: R
    (dr.AT_POST_TMU, dr.KIND_PERSIST, 0, 230, 100, (59,)),
    (dr.AT_POST_TMU, dr.KIND_PERSIST, 0, 196, 196, (62,)),
    (dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 1, 11, 100, (60,)),  # checksum memory fault
    (dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 2, 70, 5, (61,)),    # row-checksum memory fault
]


@pytest.mark.parametrize("lookahead", [True, False])
@pytest.mark.parametrize("case", range(len(CASES)))
def test_fault_campaign_parity(lib, ctx, case, lookahead):
    point, kind, target, gi, gj, bits = CASES[case]
    A = si.spd(256, seed=0)
    _compare(lib, ctx, A, 32, [dr.Inject(2, point, kind, target, gi, gj, bits)], lookahead=lookahead)


# Two faults in one iteration: the first is corrected by a pre-op check, the
# second forces the local restart of that op (L430).  The restart restores the
# op's input from the copy the pre-op check's own pass left behind
# (ft_driver.cuh check(ckpt)): that copy must hold the CORRECTED element, as
# the oracle's copy taken after the check does.
DOUBLE_CASES = [
    [(dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 0, 70, 66, (61,)), (dr.AT_PRE_PD, dr.KIND_PERSIST, 0, 75, 70, (57,))],
    [(dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 0, 200, 70, (60,)), (dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 70, 66, (60,))],
    [(dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 0, 131, 77, (59,)), (dr.AT_POST_PU, dr.KIND_PERSIST, 0, 150, 90, (63,)),
     (dr.AT_POST_PU, dr.KIND_PERSIST, 0, 155, 93, (62,))],
]


@pytest.mark.parametrize("lookahead", [True, False])
@pytest.mark.parametrize("case", range(len(DOUBLE_CASES)))
def test_restart_from_check_checkpoint(lib, ctx, case, lookahead):
    A = si.spd(256, seed=0)
    so, sg = _compare(lib, ctx, A, 32, [dr.Inject(2, *c) for c in DOUBLE_CASES[case]], lookahead=lookahead)
    assert so.restarts >= 1 and sg.restarts == so.restarts


def test_restart_from_check_checkpoint_nb1024(lib, ctx):
    """fp64 nb=1024: the locate tables do not fit the pass kernel (separate
    locate launch), and the check's copy of the PU input is patched by that
    standalone locate (abft_pass.cu run_pass)."""
    A = si.spd(4096, seed=0)
    inj = [dr.Inject(1, dr.AT_PRE_PU_CHECK, dr.KIND_PERSIST, 0, 3000, 1500, (60,)),
           dr.Inject(1, dr.AT_PRE_PU, dr.KIND_ONCHIP, 0, 1100, 1050, (60,))]
    so, sg = _compare(lib, ctx, A, 1024, inj)
    assert so.restarts == 1 and sg.restarts == 1


# fp32 (every entry point takes ABFT_F32; BASELINE's 1e-5): the same fault
# kinds with the flips moved into the fp32 word (fp64 bit b -> b - 32: the
# exponent/sign bits stay exponent/sign bits, 52-54 become mantissa 20-22)
CASES_F32 = CASES


@pytest.mark.parametrize("case", range(len(CASES_F32)))
def test_fault_campaign_parity_f32(lib, ctx, case):
    point, kind, target, gi, gj, bits = CASES_F32[case]
    A = si.spd(256, seed=0)
    _compare(lib, ctx, A, 32, [dr.Inject(2, point, kind, target, gi, gj, tuple(b - 32 for b in bits))], prec="f32")


@pytest.mark.parametrize("case", [
    # (iter, point, kind, gi, gj, bits): the metric's tile size nb=512 on n=2048
    (1, dr.AT_POST_TMU, dr.KIND_PERSIST, 1900, 1300, (60,)),   # trailing computation error -> 0D
    (1, dr.AT_PRE_TMU, dr.KIND_PERSIST, 1500, 700, (54,)),     # DRAM in the TMU reference part -> Fig. 4a repair
    (1, dr.AT_PRE_TMU, dr.KIND_ONCHIP, 1700, 600, (56,)),      # on-chip panel value during the TMU -> 1D + Fig. 4b
    (0, dr.AT_PRE_PU, dr.KIND_ONCHIP, 100, 50, (58,)),         # on-chip in L_kk during the PU -> 2D -> restart
    (2, dr.AT_PRE_PD_CHECK, dr.KIND_PERSIST, 1200, 1100, (62,)),  # DRAM in A_kk before its check
])
def test_fault_parity_nb512(lib, ctx, case):
    """One-fault driver parity against the ORACLE at the metric's nb=512
    (n=2048, 4 tile columns), not against the GPU's own fault-free run."""
    k, point, kind, gi, gj, bits = case
    A = si.spd(2048, seed=77)
    _compare(lib, ctx, A, 512, [dr.Inject(k, point, kind, 0, gi, gj, bits)])


def test_fig4a_off_matches_oracle(lib, ctx):
    A = si.spd(256, seed=0)
    so, sg = _compare(lib, ctx, A, 32, [dr.Inject(2, dr.AT_PRE_TMU, dr.KIND_PERSIST, 0, 170, 80, (54,))], fig4a=False)
    assert so.uncorrectable >= 1


def _random_plan(n, nb, seed, k_faults):
    """Seeded random single-fault-per-run plans over every hook point."""
    g = si.rng(seed)
    nt = n // nb
    plan = []
    for _ in range(k_faults):
        k = int(g.integers(0, nt - 1))
        point = int(g.integers(0, 8))
        kind = dr.KIND_ONCHIP if point in (dr.AT_PRE_PU, dr.AT_PRE_TMU) and g.random() < 0.5 else dr.KIND_PERSIST
        r0 = (k + 1) * nb
        if point in (dr.AT_PRE_PD_CHECK, dr.AT_PRE_PD, dr.AT_POST_PD):
            a, b = int(g.integers(k * nb, r0)), int(g.integers(k * nb, r0))
            gi, gj = max(a, b), min(a, b)
        elif point in (dr.AT_PRE_PU_CHECK, dr.AT_PRE_PU, dr.AT_POST_PU, dr.AT_PRE_TMU):
            gi, gj = int(g.integers(r0, n)), int(g.integers(k * nb, r0))
        else:
            a, b = int(g.integers(r0, n)), int(g.integers(r0, n))
            gi, gj = max(a, b), min(a, b)
        bit = int(g.integers(52, 64))
        plan.append(dr.Inject(k, point, kind, 0, gi, gj, (bit,)))
    return plan


@pytest.mark.parametrize("seed", range(12))
def test_random_campaign_parity(lib, ctx, seed):
    """Config-1 shape (fp64 SPD n=256 nb=32), one random fault per run at a
    random Alg. 2 hook, exponent/sign bits (MUST band)."""
    A = si.spd(256, seed=100 + seed)
    _compare(lib, ctx, A, 32, _random_plan(256, 32, seed, 1))


def test_config2_shape_error_free_and_injected(lib, ctx):
    """BASELINE configs[1]: fp64 n=10240 nb=512; error-free residual check at
    full size, then a random DRAM fault in a trailing tile, fixed."""
    n, nb = 10240, 512
    A = si.spd_device(n, seed=5)
    A0 = A.clone()
    rc, info, stats = lib.ft_potrf(ctx, A, nb)
    torch.cuda.synchronize()
    assert rc == 0 and info == 0 and list(stats.counts) == [0] * 8
    L = torch.tril(A)
    # sampled residual rows: |A0 - L L^T| on 64 random rows
    g = si.rng(9)
    rows = torch.tensor(sorted(g.choice(n, 64, replace=False)), device="cuda")
    R = A0[rows] - L[rows] @ L.T
    assert R.abs().max().item() <= 1e-12 * n
    A.copy_(A0)
    inj = [(5, lib.AT_POST_TMU, lib.KIND_PERSIST, 0, 7000, 6000, 1 << 61)]
    rc, info, stats = lib.ft_potrf(ctx, A, nb, inject=inj)
    torch.cuda.synchronize()
    assert rc == 0 and stats.counts[5] == 1
    assert (torch.tril(A) - L).abs().max().item() <= 1e-12 * L.abs().max().item()


def test_metric_size_potrf(lib, ctx):
    """The metric's ft_potrf (n=30720 nb=512, as bench.py runs it): sampled
    residual rows of the error-free factor, then one MUST-band DRAM fault in
    the trailing matrix and one on-chip fault in the panel during the TMU,
    both fixed (the factor equals the fault-free one within 1e-12)."""
    n, nb = 30720, 512
    A = si.spd_device(n, seed=6)
    A0 = A.clone()
    rc, info, stats = lib.ft_potrf(ctx, A, nb)
    torch.cuda.synchronize()
    assert rc == 0 and info == 0 and list(stats.counts) == [0] * 8
    g = si.rng(10)
    rows = torch.tensor(sorted(g.choice(n, 32, replace=False)), device="cuda")
    Lr = torch.tril(A)[rows]
    R = A0[rows] - Lr @ torch.tril(A).T
    assert R.abs().max().item() <= 1e-12 * n
    ref = torch.tril(A).clone()
    A.copy_(A0)
    inj = [(20, lib.AT_POST_TMU, lib.KIND_PERSIST, 0, 25000, 15000, 1 << 60),
           (40, lib.AT_PRE_TMU, lib.KIND_ONCHIP, 0, 29000, 20600, 1 << 55)]
    rc, info, stats = lib.ft_potrf(ctx, A, nb, inject=inj)
    torch.cuda.synchronize()
    assert rc == 0 and stats.uncorrectable == 0 and stats.n_fixes >= 2
    assert (torch.tril(A) - ref).abs().max().item() <= 1e-12 * ref.abs().max().item()


# ---- f1: Fig. 4b on-chip 1D detection and the periodic trailing check ------
_ONCHIP_PAIR = [dr.Inject(1, dr.AT_PRE_TMU, dr.KIND_ONCHIP, 0, 197, 40, (55,)),
                dr.Inject(2, dr.AT_PRE_TMU, dr.KIND_ONCHIP, 0, 212, 67, (55,))]


@pytest.mark.parametrize("fig4b,period", [(True, 0), (False, 0), (False, 1), (True, 2)])
def test_fig4b_and_periodic_parity(lib, ctx, fig4b, period):
    A_np = si.spd(256, seed=41)
    o_L, ost = dr.ft_potrf(A_np, 32, inject=_ONCHIP_PAIR, fig4b=fig4b, restart=False,
                           trailing_check_period=period, lookahead=True)
    A = dev(A_np)
    inj = [(f.iter, f.point, f.kind, f.target, f.gi, f.gj, si.mask_of(f.bits)) for f in _ONCHIP_PAIR]
    log = torch.zeros(8192 * lib.FIX_BYTES, dtype=torch.uint8, device="cuda")
    rc, info, st = lib.ft_potrf(ctx, A, 32, inject=inj, fix_log=log, restart=False, fig4b=fig4b,
                                trailing_check_period=period)
    torch.cuda.synchronize()
    fixes = lib.decode_fixes(log, st.n_fixes)
    assert (rc == lib.E_UNCORRECTABLE) == (ost.uncorrectable > 0)
    assert st.n_checks == ost.n_checks
    if ost.uncorrectable == 0:
        assert list(st.counts) == ost.counts
        assert sorted((f[0], f[1], f[4]) for f in fixes) == sorted((f.gi, f.gj, f.cls) for f in ost.fixes)
        assert np.abs(np.tril(host(A)) - o_L).max() <= 1e-12 * np.abs(o_L).max()
