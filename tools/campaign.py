"""Fault-injection campaign (BASELINE configs[0]/[1]; paper §X.A):
one random single fault per run at a random Alg. 2 hook of a random
iteration, for ft_potrf / ft_getrf / ft_geqrf on the GPU, graded as the
paper's outcomes (L580): Y = fixed (factor equals the fault-free one within
1e-12), R = detected but uncorrectable (restart needed), N = not detected /
silently wrong.  Faults use exponent/sign bits (52–63), i.e. the MUST band
of reading c-10 for O(1) elements.  Writes gpurun_out/campaign.json.

  python tools/campaign.py [trials_per_driver] [n] [nb]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

AT = dict(PRE_PD_CHECK=0, PRE_PD=1, POST_PD=2, PRE_PU_CHECK=3, PRE_PU=4, POST_PU=5, PRE_TMU=6, POST_TMU=7)


def plan(kind, n, nb, g):
    nt = n // nb
    k = int(g.integers(0, nt - 1))
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
    return (k, point, 1 if onchip else 0, 0, gi, gj, 1 << bit), bit


def main():
    trials = int(sys.argv[1]) if len(sys.argv) > 1 else 50
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
    nb = int(sys.argv[3]) if len(sys.argv) > 3 else 128
    ctx = abft.Context()
    g = si.rng(2018)
    report = {"n": n, "nb": nb, "trials": trials, "bits": "52-63"}
    for kind in ("potrf", "getrf", "geqrf"):
        A0 = si.spd_device(n, seed=1) if kind == "potrf" else si.general_device(n, seed=1)
        A = torch.empty_like(A0.t()).t()
        piv = torch.zeros(n, dtype=torch.int64, device="cuda")
        tau = torch.zeros(n, dtype=torch.float64, device="cuda")

        def run(inj):
            A.copy_(A0)
            if kind == "potrf":
                rc, info, st = abft.ft_potrf(ctx, A, nb, inject=inj)
                out = torch.tril(A).clone()
            elif kind == "getrf":
                rc, info, st = abft.ft_getrf(ctx, A, nb, piv, inject=inj)
                out = A.clone()
            else:
                rc, info, st = abft.ft_geqrf(ctx, A, nb, tau, inject=inj)
                out = A.clone()
            torch.cuda.synchronize()
            return rc, st, out

        _, _, ref = run(())
        scale = ref.abs().max().item()
        out = {"Y": 0, "R": 0, "N": 0, "detected": 0, "cases": []}
        for t in range(trials):
            inj, bit = plan(kind, n, nb, g)
            rc, st, res = run([inj])
            err = (res - ref).abs().max().item() / scale
            det = st.counts[0] > 0 or st.uncorrectable > 0
            if rc == abft.E_UNCORRECTABLE:
                o = "R"
            elif err <= 1e-12:
                o = "Y"
            else:
                o = "N"
            out[o] += 1
            out["detected"] += int(det)
            out["cases"].append({"inject": list(inj[:6]), "bit": bit, "outcome": o, "rel_err": err,
                                 "fixes": st.n_fixes, "repairs": st.repairs_applied})
        report[kind] = out
        print(kind, {k: v for k, v in out.items() if k != "cases"}, flush=True)
        del A, A0
        torch.cuda.empty_cache()
    os.makedirs("gpurun_out", exist_ok=True)
    with open("gpurun_out/campaign.json", "w") as f:
        json.dump(report, f, indent=1)


if __name__ == "__main__":
    main()
