"""Find multi-fault runs (K faults in K distinct iterations) whose GPU result
is not backward-accurate, and replay each in the CPU oracle to tell a GPU
bug (oracle fine) from an algorithmic limit (oracle equally wrong).
  python tools/multi_fault_repro.py KIND N NB K TRIALS [SEED]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from scipy.linalg import lapack

import synth_inputs as si
from oracle import drivers as dr
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

kind, n, nb, K, trials = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), int(sys.argv[5])
seed = int(sys.argv[6]) if len(sys.argv) > 6 else 5
sys.argv = sys.argv[:1]
from tools.campaign import plan  # noqa: E402

A0n = si.general(n, seed=1) if kind != "potrf" else si.spd(n, seed=1)
A0 = abft.to_colmajor(torch.from_numpy(A0n).cuda())
ctx = abft.Context()
A = torch.empty_like(A0.t()).t()
tau = torch.zeros(n, dtype=torch.float64, device="cuda")
piv = torch.zeros(n, dtype=torch.int64, device="cuda")
nA = np.linalg.norm(A0n)


def bwd_np(out, tv):
    if kind == "geqrf":
        Q, _, _ = lapack.dorgqr(np.tril(out, -1) + np.eye(n), tv)
        return np.linalg.norm(A0n - Q @ np.triu(out)) / nA
    L = np.tril(out)
    return np.linalg.norm(A0n - L @ L.T) / nA


def gpu(inj):
    A.copy_(A0)
    if kind == "geqrf":
        rc, _, st = abft.ft_geqrf(ctx, A, nb, tau, inject=inj)
    else:
        rc, _, st = abft.ft_potrf(ctx, A, nb, inject=inj)
    torch.cuda.synchronize()
    return rc, A.cpu().numpy(), tau.cpu().numpy(), st


_, ref, tref, _ = gpu(())
free = bwd_np(ref, tref)
g = si.rng(seed)
found = []
for t in range(trials):
    ks = sorted(int(x) for x in g.choice(n // nb - 1, size=K, replace=False))
    plans = [plan(kind, n, nb, g, k) for k in ks]
    inj = [p[0] for p in plans]
    rc, out, tv, st = gpu(inj)
    b = bwd_np(out, tv) if np.isfinite(out).all() else np.inf
    if rc == 0 and b > 4 * free:
        oinj = [dr.Inject(i[0], i[1], i[2], i[3], i[4], i[5], (int(i[6]).bit_length() - 1,)) for i in inj]
        if kind == "geqrf":
            oo, otau, ost = dr.ft_geqrf(A0n, nb, inject=oinj)
        else:
            oo, ost = dr.ft_potrf(A0n, nb, inject=oinj)[:2]
            otau = None
        ob = bwd_np(oo, otau) if np.isfinite(oo).all() else np.inf
        rec = {"trial": t, "inject": [list(map(int, i[:6])) + [int(i[6]).bit_length() - 1] for i in inj],
               "gpu_bwd": b, "free_bwd": free, "gpu_fixes": st.n_fixes, "oracle_bwd": ob,
               "oracle_uncorrectable": int(ost.uncorrectable), "oracle_fixes": len(ost.fixes),
               "gpu_vs_oracle": float(np.abs(np.tril(out) - np.tril(oo)).max() / np.abs(oo).max())}
        found.append(rec)
        print(json.dumps(rec), flush=True)
print(json.dumps({"kind": kind, "n": n, "nb": nb, "K": K, "trials": trials, "found": len(found), "free_bwd": free}))
