"""Row f4: the coverage probability model (paper §X.B, reading c-33) —
host-side analysis, CPU only.  Pins: the event probabilities are binomial
pmfs (scipy.stats.binom), outcomes of one op partition probability one,
first-order limits, the scheme tables order as the paper's protection
analysis says (ours never worse, strictly better somewhere)."""
import math

import pytest
from scipy.stats import binom

from paper_conf_sc_chenlllwtolzgc18_b200 import coverage as cv


@pytest.mark.parametrize("n,p", [(10, 0.01), (1000, 1e-4), (12345, 3e-6)])
def test_none_and_one_are_binomial(n, p):
    assert math.isclose(cv.p_none(n, p), binom.pmf(0, n, p), rel_tol=1e-12)
    assert math.isclose(cv.p_one(n, p), binom.pmf(1, n, p), rel_tol=1e-12)


def test_first_order_limit_and_zero_rates():
    n, p = 1e12, 1e-20
    assert math.isclose(cv.p_one(n, p), n * p, rel_tol=1e-6)
    assert math.isclose(1.0 - cv.p_none(n, p), n * p, rel_tol=1e-6)
    op = cv.cholesky_iteration(10240, 256, 1e-4, 1e-3, 2e-2)["TMU"]
    o = cv.outcomes("TMU", op, cv.Rates(0, 0, 0, 0), "ours")
    assert o["fault_free"] == 1.0 and o[cv.Y] == o[cv.R] == o[cv.N] == 0.0


@pytest.mark.parametrize("it", [cv.cholesky_iteration, cv.lu_iteration])
@pytest.mark.parametrize("scheme", cv.SCHEMES)
def test_outcomes_partition_one(it, scheme):
    ops = it(10240, 256, 2e-4, 1e-3, 3e-2)
    rates = cv.Rates(1e-13, 1e-6, 1e-6, 1e-9)  # large enough that faults matter
    for name, op in ops.items():
        o = cv.outcomes(name, op, rates, scheme)
        assert all(v >= 0 for v in o.values())
        assert math.isclose(sum(o.values()), 1.0, rel_tol=1e-12)
        e = cv.event_probabilities(op, rates)
        assert math.isclose(e["fault_free"] + sum(e["single"].values()) + o["multi"], 1.0, rel_tol=1e-12)


def test_tables_complete_and_ours_dominates():
    rank = {cv.Y: 0, cv.R: 1, cv.N: 2}
    strictly = 0
    for s in cv.SCHEMES:
        for op in cv.OPS:
            assert set(cv.OUTCOME[s][op]) == set(cv.FAULTS)
    for s in cv.SCHEMES:
        for op in cv.OPS:
            for f in cv.FAULTS:
                a, b = rank[cv.OUTCOME["ours"][op][f]], rank[cv.OUTCOME[s][op][f]]
                assert a <= b, (s, op, f)
                strictly += a < b
    assert strictly > 0
    # the paper's specific claims: single-side cannot tolerate PU faults (L584),
    # only the post-broadcast check catches PCIe faults (L346, L355)
    assert cv.OUTCOME["single_prior"]["PU"]["comp"] == cv.N
    assert all(cv.OUTCOME[s][op]["pcie"] == cv.N for s in cv.SCHEMES[:3] for op in cv.OPS)


def test_expected_recovery_ours_lowest():
    ops = cv.lu_iteration(10240, 256, 2e-4, 1e-3, 3e-2)
    rates = cv.Rates()
    cost = {s: sum(cv.expected_recovery_time(n, op, rates, s, t_fix=1e-5, t_total=1.0) for n, op in ops.items())
            for s in cv.SCHEMES}
    assert cost["ours"] == min(cost.values()) and cost["ours"] < cost["single_prior"]


def _campaigns():
    import json
    import os

    root = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles")
    out = []
    for f in sorted(os.listdir(root)):
        if "campaign_n" in f and f.endswith(".json") and "schemes" not in f:
            with open(os.path.join(root, f)) as fh:
                out.append(json.load(fh))
    return out


def test_ours_row_agrees_with_the_measured_campaigns():
    """The 'ours' row is generated from the committed campaigns wherever they
    sampled a cell: the reading's entry is the most frequent measured
    outcome, and no campaign run ended silently wrong."""
    frac, runs = cv.campaign_fractions(_campaigns())
    assert frac, "no campaign JSON under profiles/"
    seen = 0
    for op, cells in frac.items():
        for f, d in cells.items():
            assert abs(sum(d.values()) - 1.0) < 1e-12
            top = max(d, key=d.get)
            assert cv.OUTCOME["ours"][op][f] == top, (op, f, d, runs[op][f])
            seen += 1
    assert seen >= 9  # PD / PU / TMU cells the campaigns draw (+ the PD transfers)
    o = cv.outcomes("TMU", cv.lu_iteration(10240, 256, 2e-4, 1e-3, 3e-2)["TMU"], cv.Rates(1e-13, 1e-6, 1e-6, 1e-9),
                    "ours", frac)
    assert math.isclose(sum(o.values()), 1.0, rel_tol=1e-12)
