"""Row f4 on B200: the coverage model (paper §X.B, Figs. 6-11's setting:
one iteration of LU — and Cholesky — with n=10240, nb=256, the paper's
illustrative rates, L640-L645) evaluated with operation times A_OP measured
here (cuSOLVER / cuBLAS through torch, CUDA events, median of 20).
Writes gpurun_out/coverage.json.

  python tools/coverage_eval.py [n] [nb]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_sc_chenlllwtolzgc18_b200 import coverage as cv


def timed(fn, reps=20):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / 1e3)
    return sorted(ts)[reps // 2]


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 10240
    nb = int(sys.argv[2]) if len(sys.argv) > 2 else 256
    torch.backends.cuda.preferred_linalg_library("cusolver")
    g = torch.Generator(device="cuda").manual_seed(0)
    m = n - nb
    M = torch.rand(n, n, device="cuda", dtype=torch.float64, generator=g)
    S = (M[:nb, :nb] + M[:nb, :nb].T) / 2 + nb * torch.eye(nb, device="cuda", dtype=torch.float64)
    L = torch.linalg.cholesky(S)
    panel = M[:, :nb].contiguous()
    A21 = M[nb:, :nb].contiguous()
    A12 = M[:nb, nb:].contiguous()
    A22 = M[nb:, nb:].contiguous()
    times = {
        "chol": {"PD": timed(lambda: torch.linalg.cholesky(S)),
                 "PU": timed(lambda: torch.linalg.solve_triangular(L, A21.T, upper=False)),
                 "TMU": timed(lambda: torch.addmm(A22, A21, A21.T, beta=1.0, alpha=-1.0))},
        "lu": {"PD": timed(lambda: torch.linalg.lu_factor(panel)),
               "PU": timed(lambda: torch.linalg.solve_triangular(L, A12, upper=False, unitriangular=True)),
               "TMU": timed(lambda: torch.addmm(A22, A21, A12, beta=1.0, alpha=-1.0))},
    }
    rates = cv.Rates()
    # "ours" generated from the committed single-fault campaigns (outcome
    # fractions per op / fault, tools/campaign.py); unsampled cells: the table
    prof = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles")
    camps = []
    for f in sorted(os.listdir(prof)):
        if "campaign_n" in f and f.endswith(".json") and "schemes" not in f:
            with open(os.path.join(prof, f)) as fh:
                camps.append(json.load(fh))
    measured, runs = cv.campaign_fractions(camps)
    out = {"n": n, "nb": nb, "rates": vars(rates), "a_op_s": times, "device": torch.cuda.get_device_name(),
           "ours_measured_fractions": measured, "ours_measured_runs": runs,
           "note": "one iteration at n_k = n; t_fix = 1e-5 s; complete restart = sum of the iteration's ops x n/nb; "
                   "'ours' uses the campaigns' outcome fractions where they sampled the cell"}
    for name, it in (("chol", cv.cholesky_iteration), ("lu", cv.lu_iteration)):
        t = times[name]
        ops = it(n, nb, t["PD"], t["PU"], t["TMU"])
        t_total = (t["PD"] + t["PU"] + t["TMU"]) * (n // nb) / 3.0  # ~ n/nb iterations shrinking cubically
        res = {}
        for s in cv.SCHEMES:
            res[s] = {op: {k: v for k, v in cv.outcomes(op, ops[op], rates, s, measured).items()} for op in cv.OPS}
            res[s]["expected_recovery_s"] = sum(
                cv.expected_recovery_time(op, ops[op], rates, s, 1e-5, t_total, measured) for op in cv.OPS)
        out[name] = res
        print(name, {s: res[s]["expected_recovery_s"] for s in cv.SCHEMES}, flush=True)
    os.makedirs("gpurun_out", exist_ok=True)
    with open("gpurun_out/coverage.json", "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
