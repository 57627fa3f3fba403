"""Fault-injection campaign (BASELINE configs[0]/[1]; paper §X.A):
one random single fault per run at a random Alg. 2 hook of a random
iteration, for ft_potrf / ft_getrf / ft_geqrf on the GPU, graded as the
paper's outcomes (L580): Y = fixed (factor equals the fault-free one within
1e-12; "restarts" counts the runs that needed the local restart, f1),
R = detected but uncorrectable (complete restart needed), N = not detected /
silently wrong.  Faults use exponent/sign bits (52–63), i.e. the MUST band
of reading c-10 for O(1) elements.  QR runs also draw faults in the CTF T
(f2); a fourth campaign, "host", runs ft_potrf / ft_getrf with the PD on the
host (FT_PD_HOST) and draws D2H / H2D transfer faults (Alg. 2 lines 3, 6).
With K > 1 faults per run (BASELINE configs[1]: K in {1, 2, 4}), the K
faults hit K distinct iterations and K distinct tiles, so at most one fault
lands in a tile between two checks (L275).  Grading per fault kind (reading c-10): a run
whose faults are all outside the TMU reference part must end Y; a run with a
TMU reference-part fault (PRE_TMU hook: memory or on-chip in a panel tile the
TMU reads) must end Y or R; N fails every run.
"Correct final result" (the paper's Y vs N, L580) is judged by backward
error, not by equality with the fault-free factor: a corrected element is
exact only to its checksum's rounding (reading c-4, <= tau), and LU / QR
amplify such a perturbation in the forward factors (pivot growth) while the
factorization stays backward stable.  Y: rc == 0 and ||A - factors||_F /
||A||_F <= 4x the fault-free run's; Yr ("rounding residue"): above that but
within LAPACK's own acceptance test for a factorization, ratio
||A - factors|| / (||A|| n u) <= 30 (the threshold of LAPACK's xCHKPO /
xCHKGE / xCHKQR test drivers) — many corrections, each exact only to tau,
add up; N: beyond.  The forward deviation from the fault-free factor is
reported beside it (rel_err).
Writes gpurun_out/campaign.json (or the path in $CAMPAIGN_OUT).

Kinds potrf:full_post, potrf:single_post, potrf:single_pre run ft_potrf
with the other checking schemes the paper compares (L542, Table VIII;
ft_opts_t.scheme, reading c-34) on the same fault draws.

  python tools/campaign.py [trials_per_driver] [n] [nb] [K,K,..] [kind,kind,..]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

AT = dict(PRE_PD_CHECK=0, PRE_PD=1, POST_PD=2, PRE_PU_CHECK=3, PRE_PU=4, POST_PU=5, PRE_TMU=6, POST_TMU=7,
          D2H=8, H2D=9)


def plan(kind, n, nb, g, k=None):
    nt = n // nb
    k = int(g.integers(0, nt - 1)) if k is None else k
    r0, r1 = k * nb, (k + 1) * nb
    if kind == "potrf":
        point = int(g.integers(0, 8))
    elif kind == "getrf":
        point = int(g.integers(0, 8))
    else:
        point = [0, 2, 6, 7][int(g.integers(0, 4))]
    onchip = point in (AT["PRE_PU"], AT["PRE_TMU"]) and g.random() < 0.5
    if kind == "potrf":
        if point <= 2:
            a, b = int(g.integers(r0, r1)), int(g.integers(r0, r1))
            gi, gj = max(a, b), min(a, b)
        elif point <= 6:
            gi, gj = int(g.integers(r1, n)), int(g.integers(r0, r1))
        else:
            a, b = int(g.integers(r1, n)), int(g.integers(r1, n))
            gi, gj = max(a, b), min(a, b)
    else:
        if point <= 2:
            gi, gj = int(g.integers(r0, n)), int(g.integers(r0, r1))
        elif point <= 5:
            gi, gj = int(g.integers(r0, r1)), int(g.integers(r1, n))
        elif point == 6:
            gi, gj = (int(g.integers(r1, n)), int(g.integers(r0, r1))) if g.random() < 0.5 else \
                (int(g.integers(r0, r1)), int(g.integers(r1, n)))
        else:
            gi, gj = int(g.integers(r1, n)), int(g.integers(r1, n))
    bit = int(g.integers(52, 64))
    target = 0
    if kind == "geqrf" and point == AT["POST_PD"] and g.random() < 0.25:  # CTF T (f2)
        target, gi, gj = 3, int(g.integers(0, nb)), int(g.integers(0, nb))
        gi, gj = min(gi, gj), max(gi, gj)  # upper triangle incl. the diagonal
    if kind.startswith("host"):
        point = AT["D2H"] if g.random() < 0.5 else AT["H2D"]
        onchip = False
        rows = nb if kind == "host_potrf" else n - r0
        gi, gj = r0 + int(g.integers(0, rows)), int(g.integers(r0, r1))
        if kind == "host_potrf":
            a, b = gi, gj
            gi, gj = max(a, b), min(a, b)
    return (k, point, 1 if onchip else 0, target, gi, gj, 1 << bit), bit


def main():
    trials = int(sys.argv[1]) if len(sys.argv) > 1 else 50
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
    nb = int(sys.argv[3]) if len(sys.argv) > 3 else 128
    Ks = [int(x) for x in sys.argv[4].split(",")] if len(sys.argv) > 4 else [1]
    kinds = sys.argv[5].split(",") if len(sys.argv) > 5 else ["potrf", "getrf", "geqrf", "host_potrf", "host_getrf"]
    ctx = abft.Context()
    ctx.set_host_lapack()
    g = si.rng(2018)
    report = {"n": n, "nb": nb, "trials": trials, "bits": "52-63", "K": Ks}
    SCHEME = {"": abft.SCHEME_NEW, "full_post": abft.SCHEME_FULL_POST, "single_post": abft.SCHEME_SINGLE_POST,
              "single_pre": abft.SCHEME_SINGLE_PRE}
    for label, K in [(kd, K) for kd in kinds for K in Ks]:
        kind, _, sname = label.partition(":")
        scheme = SCHEME[sname]
        g = si.rng(2018 + K)  # every driver / scheme sees the same draw sequence for a given K
        pd = abft.PD_HOST if kind.startswith("host") else abft.PD_DEVICE
        A0 = si.spd_device(n, seed=1) if kind.endswith("potrf") else si.general_device(n, seed=1)
        A = torch.empty_like(A0.t()).t()
        piv = torch.zeros(n, dtype=torch.int64, device="cuda")
        tau = torch.zeros(n, dtype=torch.float64, device="cuda")

        nA = torch.linalg.norm(A0).item()

        def resid(out):
            """||A0 - factors||_F / ||A0||_F (backward error of the run's output)."""
            if kind.endswith("potrf"):
                return torch.linalg.norm(A0 - out @ out.t()).item() / nA
            if kind.endswith("getrf"):
                perm = np.arange(n)
                for i, p in enumerate(piv.cpu().numpy() - 1):
                    perm[i], perm[p] = perm[p], perm[i]
                L = torch.tril(out, -1) + torch.eye(n, dtype=out.dtype, device=out.device)
                return torch.linalg.norm(A0[torch.from_numpy(perm).cuda()] - L @ torch.triu(out)).item() / nA
            Q = torch.linalg.householder_product(torch.tril(out, -1), tau)
            return torch.linalg.norm(A0 - Q @ torch.triu(out)).item() / nA

        def run(inj):
            A.copy_(A0)
            if kind.endswith("potrf"):
                rc, info, st = abft.ft_potrf(ctx, A, nb, inject=inj, pd_location=pd, scheme=scheme)
                out = torch.tril(A).clone()
            elif kind.endswith("getrf"):
                rc, info, st = abft.ft_getrf(ctx, A, nb, piv, inject=inj, pd_location=pd)
                out = A.clone()
            else:
                rc, info, st = abft.ft_geqrf(ctx, A, nb, tau, inject=inj)
                out = A.clone()
            torch.cuda.synchronize()
            return rc, st, out

        _, st0, ref = run(())
        free_ms = sorted([st0.ms_total] + [run(())[1].ms_total for _ in range(2)])[1]
        scale = ref.abs().max().item()
        res_free = resid(ref)
        out = {"K": K, "backward_err_fault_free": res_free, "Y": 0, "Yr": 0, "R": 0, "N": 0, "detected": 0, "restarts": 0, "graded_pass": 0, "cases": []}
        for t in range(trials):
            while True:  # K distinct iterations AND K distinct tiles (a trailing tile hit at
                # iteration k may be checked first many iterations later: two faults in it
                # before that check would break the one-fault-per-tile model, L275)
                ks = sorted(int(x) for x in g.choice(n // nb - 1, size=K, replace=False))
                plans = [plan(kind, n, nb, g, k) for k in ks]
                tiles = {(p[0][4] // nb, p[0][5] // nb) for p in plans}
                if len(tiles) == K:
                    break
            inj = [p[0] for p in plans]
            bit = [p[1] for p in plans]
            rc, st, res = run(inj)
            err = (res - ref).abs().max().item() / scale
            bwd = resid(res) if torch.isfinite(res).all() else float("inf")
            det = (st.counts[0] > 0 or st.uncorrectable > 0 or st.restarts > 0 or st.ctf_flagged > 0
                   or st.xfer_d2h_flagged > 0 or st.xfer_h2d_flagged > 0)
            if rc == abft.E_UNCORRECTABLE:
                o = "R"
            elif bwd <= 4 * res_free:
                o = "Y"
            elif bwd <= 30 * n * 2.0 ** -53:
                o = "Yr"
            else:
                o = "N"
            out[o] += 1
            out["detected"] += int(det)
            out["restarts"] += int(st.restarts > 0)
            tmu_ref = any(i[1] == AT["PRE_TMU"] for i in inj)
            out["graded_pass"] += int(o in ("Y", "Yr") or (o == "R" and tmu_ref))
            out["cases"].append({"inject": [list(i[:6]) for i in inj], "bit": bit, "outcome": o, "rel_err": err,
                                 "recovery_overhead_pct": 100.0 * (st.ms_total - free_ms) / free_ms,
                                 "backward_err": bwd,
                                 "tmu_ref": tmu_ref,
                                 "fixes": st.n_fixes, "repairs": st.repairs_applied, "restarts": st.restarts,
                                 "ctf": st.ctf_recomputed, "xfer_fixed": st.xfer_d2h_fixed + st.xfer_h2d_fixed,
                                 "retransfers": st.xfer_retransfers + st.xfer_resends})
        # recovery cost (Table VIII's overhead columns, L580): run time with the
        # fault(s) vs the fault-free protected run, per outcome
        rec = {}
        for o in ("Y", "Yr", "R"):
            v = sorted(c["recovery_overhead_pct"] for c in out["cases"] if c["outcome"] == o)
            if v:
                rec[o] = {"median_pct": v[len(v) // 2], "max_pct": v[-1]}
        v = sorted(c["recovery_overhead_pct"] for c in out["cases"] if c["outcome"] == "Y" and c["restarts"])
        if v:
            rec["Y_with_restart"] = {"median_pct": v[len(v) // 2], "max_pct": v[-1]}
        out["recovery_overhead"] = rec
        out["fault_free_ms"] = free_ms
        report[label if len(Ks) == 1 else f"{label}_K{K}"] = out
        print(label, {k: v for k, v in out.items() if k != "cases"}, flush=True)
        del A, A0
        torch.cuda.empty_cache()
    os.makedirs("gpurun_out", exist_ok=True)
    with open(os.environ.get("CAMPAIGN_OUT", "gpurun_out/campaign.json"), "w") as f:
        json.dump(report, f, indent=1)


if __name__ == "__main__":
    main()
