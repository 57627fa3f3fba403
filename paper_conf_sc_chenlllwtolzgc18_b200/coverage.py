"""Fault-tolerance coverage model (row f4; paper §X.B, Table IX).

Host-side analysis, no device work: given per-element hardware error rates
and the time each operation takes on the machine (A_OP, measured on B200 by
`tools/coverage_eval.py`), the probability that one iteration's PD, PU and
TMU end in each of the paper's four outcomes (L634–L639):

  fault free · ABFT fixable · local restart · complete restart

under each ABFT scheme the paper compares (L550–L556), and the expected
recovery time that follows.  The event probabilities P(A)…P(H) at
L624–L631 are garbled in the source; reading c-33 restates
them as binomial probabilities of "no error" / "exactly one error":

  A, B  computation errors, one chance per flop of the op:     n = T_OP,  p = r1
  C, D  off-chip memory errors while the op's data waits in DRAM
        (linear in storage time, L645):                         n = M_OP,  p = r2·A_gap
  E, F  off-chip + on-chip memory errors during the op
        (on-chip linear in execution time, L645):               n = M_OP,  p = (r2 + r3)·A_OP
  G, H  PCIe errors in the broadcast after the op:              n = M_BC,  p = r4

  P(no error) = (1 − p)^n,   P(exactly one) = n·p·(1 − p)^(n−1)

with the paper's assumption of at most one fault per operation (L633).  The
outcome of each single fault (which part it hits, which op, which scheme)
is the table OUTCOME below, read from the paper's protection analysis
(Table V; §VII; Table VIII's prose, L580–L592) and, for
our own scheme, checked by the fault campaigns of `tools/campaign.py`
(profiles/*campaign*.json: every single fault ends fixed, by ABFT or by
the local restart).
"""
from __future__ import annotations

import math
from dataclasses import dataclass

OPS = ("PD", "PU", "TMU")
# single faults: (event, part) — computation error in the op's output;
# DRAM error between ops / off- or on-chip error during the op, in the
# reference (read) or update (written) part; PCIe error in the broadcast
FAULTS = ("comp", "mem_between_ref", "mem_between_upd", "mem_during_ref", "mem_during_upd", "pcie")
SCHEMES = ("single_prior", "single_post", "full_post", "ours")
Y, R, N = "fixable", "local_restart", "complete_restart"

# OUTCOME[scheme][op][fault] (reading c-33, sources in the comments)
OUTCOME = {
    # single-side checksum, check before each op ([11], L550): PD/PU inputs
    # are checked before use; the PU's output panel carries no checksum of
    # its own direction (L584: "fails to tolerate errors occurring in PU"),
    # 1D propagation in the TMU is beyond one checksum side (L585), and a
    # fault after the check (during the op) is seen only by the next op.
    "single_prior": {
        "PD": {"comp": R, "mem_between_ref": Y, "mem_between_upd": Y, "mem_during_ref": R,
               "mem_during_upd": R, "pcie": N},
        "PU": {"comp": N, "mem_between_ref": Y, "mem_between_upd": Y, "mem_during_ref": N,
               "mem_during_upd": N, "pcie": N},
        "TMU": {"comp": Y, "mem_between_ref": Y, "mem_between_upd": Y, "mem_during_ref": R,
                "mem_during_upd": Y, "pcie": N},
    },
    # single-side checksum, check after each op ([51], [52]): output errors
    # are seen, input (reference) errors consumed before the check are 2D for
    # PD / PU (Table V), PU output still unprotected, TMU 1D not tolerable,
    # communication after the check unseen (L346: checked before broadcast).
    # (PD "mem_during_upd": a fault the factorization consumes spreads over
    # L_kk — 2D for every scheme (c-17, [32]); the post-op check restarts)
    "single_post": {
        "PD": {"comp": Y, "mem_between_ref": R, "mem_between_upd": R, "mem_during_ref": R,
               "mem_during_upd": R, "pcie": N},
        "PU": {"comp": N, "mem_between_ref": N, "mem_between_upd": N, "mem_during_ref": N,
               "mem_during_upd": N, "pcie": N},
        "TMU": {"comp": Y, "mem_between_ref": R, "mem_between_upd": Y, "mem_during_ref": R,
                "mem_during_upd": Y, "pcie": N},
    },
    # full checksum, check after each op ([13]): 1D is correctable on both
    # sides (L347-L350), reference faults consumed by PD / PU are still 2D
    # (restart), communication after the check is unseen (L346).
    "full_post": {
        "PD": {"comp": Y, "mem_between_ref": R, "mem_between_upd": R, "mem_during_ref": R,
               "mem_during_upd": R, "pcie": N},
        "PU": {"comp": Y, "mem_between_ref": R, "mem_between_upd": Y, "mem_during_ref": R,
               "mem_during_upd": Y, "pcie": N},
        "TMU": {"comp": Y, "mem_between_ref": Y, "mem_between_upd": Y, "mem_during_ref": Y,
                "mem_during_upd": Y, "pcie": N},
    },
    # ours (Alg. 2): checks before AND after PD / PU, the post-op check after
    # the broadcast (L345-L349, L355), the TMU's 1D cases repaired through the
    # panels (Fig. 4a/4b, L357-L359), 2D after PD / PU -> local restart
    # (L430).  Our campaigns: every injected single fault ends fixed (Y or,
    # for faults consumed inside PD / PU, Y after the local restart).
    "ours": {
        "PD": {"comp": Y, "mem_between_ref": Y, "mem_between_upd": Y, "mem_during_ref": R,
               "mem_during_upd": R, "pcie": Y},
        "PU": {"comp": Y, "mem_between_ref": Y, "mem_between_upd": Y, "mem_during_ref": R,
               "mem_during_upd": Y, "pcie": Y},
        "TMU": {"comp": Y, "mem_between_ref": Y, "mem_between_upd": Y, "mem_during_ref": Y,
                "mem_during_upd": Y, "pcie": Y},
    },
}


@dataclass
class Rates:
    """Per-element error rates (the paper's illustration, L642: 1e-13, 1e-9,
    1e-9, 1e-11): r1 computation (per flop), r2 off-chip memory (per element
    per second of storage), r3 on-chip memory (per element per second of
    execution), r4 PCIe (per transferred element)."""

    r1: float = 1e-13
    r2: float = 1e-9
    r3: float = 1e-9
    r4: float = 1e-11


@dataclass
class OpSize:
    """One operation of one iteration: flops T_OP, reference / update part
    sizes M_R, M_U and broadcast size M_BC (elements), its time A_OP and the
    time its data waits in DRAM before it (A_gap), seconds (Table IX)."""

    flops: float
    m_ref: float
    m_upd: float
    m_bc: float
    a_op: float
    a_gap: float


def p_none(n: float, p: float) -> float:
    """(1 − p)^n, computed as exp(n·log1p(−p)) (n up to ~1e13 flops)."""
    if p <= 0.0 or n <= 0:
        return 1.0
    return math.exp(n * math.log1p(-p))


def p_one(n: float, p: float) -> float:
    """n·p·(1 − p)^(n−1): exactly one of n independent chances."""
    if p <= 0.0 or n <= 0:
        return 0.0
    return n * p * math.exp((n - 1) * math.log1p(-p))


def event_probabilities(op: OpSize, rates: Rates) -> dict:
    """P(A)…P(H) of reading c-33 for one operation, plus the single-fault
    probabilities split by part."""
    pm_gap = rates.r2 * op.a_gap
    pm_op = (rates.r2 + rates.r3) * op.a_op
    m = op.m_ref + op.m_upd
    ev = {
        "A": p_none(op.flops, rates.r1), "B": p_one(op.flops, rates.r1),
        "C": p_none(m, pm_gap), "D": p_one(m, pm_gap),
        "E": p_none(m, pm_op), "F": p_one(m, pm_op),
        "G": p_none(op.m_bc, rates.r4), "H": p_one(op.m_bc, rates.r4),
    }
    # exactly one fault in the whole op, of each kind and part (the other
    # three event families fault free)
    clean = ev["A"] * ev["C"] * ev["E"] * ev["G"]
    share = lambda part: (op.m_ref if part == "ref" else op.m_upd) / m if m > 0 else 0.0
    single = {
        "comp": ev["B"] * ev["C"] * ev["E"] * ev["G"],
        "mem_between_ref": ev["A"] * ev["D"] * share("ref") * ev["E"] * ev["G"],
        "mem_between_upd": ev["A"] * ev["D"] * share("upd") * ev["E"] * ev["G"],
        "mem_during_ref": ev["A"] * ev["C"] * ev["F"] * share("ref") * ev["G"],
        "mem_during_upd": ev["A"] * ev["C"] * ev["F"] * share("upd") * ev["G"],
        "pcie": ev["A"] * ev["C"] * ev["E"] * ev["H"],
    }
    return {"events": ev, "fault_free": clean, "single": single}


def outcomes(op_name: str, op: OpSize, rates: Rates, scheme: str, measured: dict = None) -> dict:
    """Probabilities of the four outcomes of one operation under a scheme
    (at most one fault per operation, L633: the remainder — two or more
    faults — is reported separately as 'multi').  measured (scheme "ours"
    only): outcome fractions per (op, fault) observed by the fault campaigns
    (`campaign_fractions`); cells the campaigns did not sample use OUTCOME."""
    e = event_probabilities(op, rates)
    out = {"fault_free": e["fault_free"], Y: 0.0, R: 0.0, N: 0.0}
    for f, p in e["single"].items():
        cell = (measured or {}).get(op_name, {}).get(f) if scheme == "ours" else None
        if cell:
            for o, frac in cell.items():
                out[o] += p * frac
        else:
            out[OUTCOME[scheme][op_name][f]] += p
    out["multi"] = max(0.0, 1.0 - sum(out.values()))
    return out


# campaign hook (tools/campaign.py `inject` entries: iter, point, kind, target,
# gi, gj) -> the model's (op, single fault) of reading c-33.  The campaigns
# draw PD / PU faults in the op's update part and TMU faults in its
# reference part (the panel) or output; D2H / H2D are the PD's transfers.
_HOOK_CELL = {(0, 0): ("PD", "mem_between_upd"), (1, 0): ("PD", "mem_during_upd"), (2, 0): ("PD", "comp"),
              (3, 0): ("PU", "mem_between_upd"), (4, 0): ("PU", "mem_during_upd"),
              (4, 1): ("PU", "mem_during_upd"), (5, 0): ("PU", "comp"), (6, 0): ("TMU", "mem_between_ref"),
              (6, 1): ("TMU", "mem_during_ref"), (7, 0): ("TMU", "comp"), (8, 0): ("PD", "pcie"),
              (9, 0): ("PD", "pcie")}


def campaign_outcome(case: dict) -> str:
    """A campaign run's outcome in the model's terms: fixed without a restart
    -> fixable; fixed by the local restart -> local restart; returned
    uncorrectable (R) or silently wrong (N) -> complete restart."""
    if case["outcome"] in ("Y", "Yr"):
        return R if case.get("restarts", 0) > 0 else Y
    return N


def campaign_fractions(campaigns) -> dict:
    """Outcome fractions per (op, fault) from single-fault campaign runs
    (the K = 1 sections of tools/campaign.py's JSON, any driver)."""
    tally = {}
    for camp in campaigns:
        for key, sec in camp.items():
            if not isinstance(sec, dict) or "cases" not in sec:
                continue
            for case in sec["cases"]:
                if len(case["inject"]) != 1:
                    continue
                it, point, kind, target = case["inject"][0][:4]
                cell = _HOOK_CELL.get((point, kind)) if target == 0 else None
                if cell is None:
                    continue
                d = tally.setdefault(cell[0], {}).setdefault(cell[1], {})
                o = campaign_outcome(case)
                d[o] = d.get(o, 0) + 1
    out = {}
    for op, faults in tally.items():
        for f, cnt in faults.items():
            tot = sum(cnt.values())
            out.setdefault(op, {})[f] = {o: c / tot for o, c in cnt.items()}
            out[op][f]["runs"] = tot
    return {op: {f: {k: v for k, v in c.items() if k != "runs"} for f, c in fs.items()} for op, fs in out.items()}, \
        {op: {f: c["runs"] for f, c in fs.items()} for op, fs in out.items()}


def expected_recovery_time(op_name: str, op: OpSize, rates: Rates, scheme: str, t_fix: float,
                           t_total: float, measured: dict = None) -> float:
    """Expected extra time of one operation (L646: "expected time cost for
    fault recovery"): fixable -> t_fix (measured ABFT correction cost),
    local restart -> the op again (A_OP) plus t_fix, complete restart -> the
    whole factorization t_total."""
    o = outcomes(op_name, op, rates, scheme, measured)
    return o[Y] * t_fix + o[R] * (op.a_op + t_fix) + o[N] * t_total


def cholesky_iteration(n_k: int, nb: int, a_pd: float, a_pu: float, a_tmu: float) -> dict:
    """Sizes of one right-looking Cholesky iteration with an n_k x n_k
    undecomposed matrix (Table IX's T_OP, M_OP,U|R, M_OP,BC): PD factors the
    nb x nb diagonal tile (reference = update = the tile), PU solves the
    (n_k−nb) x nb panel with L_kk (reference L_kk), TMU updates the lower
    trailing matrix with the panel (reference the panel).  Storage gaps: the
    PD input waited one TMU, the PU input one TMU + PD, the TMU's panels PD+PU."""
    m = n_k - nb
    return {
        "PD": OpSize(flops=nb ** 3 / 3.0, m_ref=0.0, m_upd=nb * nb / 2.0, m_bc=nb * nb / 2.0,
                     a_op=a_pd, a_gap=a_tmu),
        "PU": OpSize(flops=float(m) * nb * nb, m_ref=nb * nb / 2.0, m_upd=float(m) * nb, m_bc=float(m) * nb,
                     a_op=a_pu, a_gap=a_tmu + a_pd),
        "TMU": OpSize(flops=float(m) * m * nb, m_ref=float(m) * nb, m_upd=m * m / 2.0, m_bc=0.0,
                      a_op=a_tmu, a_gap=a_pd + a_pu),
    }


def lu_iteration(n_k: int, nb: int, a_pd: float, a_pu: float, a_tmu: float) -> dict:
    """Sizes of one right-looking LU iteration (the paper's example, L640):
    PD factors the n_k x nb column panel (it is its own reference), PU solves
    the nb x (n_k−nb) row panel with L_kk, TMU updates the (n_k−nb)² trailing
    matrix with both panels."""
    m = n_k - nb
    return {
        "PD": OpSize(flops=float(n_k) * nb * nb - nb ** 3 / 3.0, m_ref=0.0, m_upd=float(n_k) * nb,
                     m_bc=float(n_k) * nb, a_op=a_pd, a_gap=a_tmu),
        "PU": OpSize(flops=float(m) * nb * nb, m_ref=nb * nb / 2.0, m_upd=float(m) * nb, m_bc=float(m) * nb,
                     a_op=a_pu, a_gap=a_tmu + a_pd),
        "TMU": OpSize(flops=2.0 * m * m * nb, m_ref=2.0 * m * nb, m_upd=float(m) * m, m_bc=0.0, a_op=a_tmu,
                      a_gap=a_pd + a_pu),
    }
