"""Exhaustive single-flip campaign at BASELINE configs[0] (SURVEY §4
'brute-force flips', §8c c-10; north_star: "100% detection, location and
correction of injected single errors per tile").

fp64 SPD n=256 nb=32 (and the same shape in fp32), SYM_LOWER lower-only
tiles with full checksums, fresh encode.  Every stored element of every
lower tile x every bit of its IEEE word is flipped once; each trial flips the
same local (i, j, bit) in all 36 lower tiles at once (one fault per tile
between two checks, L275), then runs abft_verify + abft_locate_correct
through the C ABI.  Diagonal tiles take only their stored lower triangle.

Grading (reading c-10, extended to full checksums: the band uses every
checksum vector the flip touches — the stored column and row, and for a
diagonal tile also the mirrored column and row of the symmetric view):
  MUST      |delta| >= 16*nb*max(tau_e) or non-finite: the tile is flagged,
            exactly one data fix at the flipped element, class 0D, value
            restored within tau_e of the original, nothing else changed;
  NEED-NOT  |delta| <= min(tau_e)/8: the tile is not flagged, nothing changes;
  GRAY      otherwise: outcomes counted and reported, not graded.
tau_e = 2*gamma_nb*m with m = e^T|X| of the error-free state (c-6).

Oracle parity on a stratified sample (4 trials per bit): per tile outside
GRAY, status after verify and after locate, fix records (position, class,
kind) bit-exact, corrected data within 1e-12 (fp64) / 1e-5 (fp32).
"""
import json
import os

import numpy as np
import pytest
import torch

import synth_inputs as si
from oracle import checksum as ck
from tests.gpu_helpers import dev, host

pytestmark = pytest.mark.gpu

N, NB = 256, 32
NT = N // NB
FIX_DT = np.dtype([("gi", "<i8"), ("gj", "<i8"), ("before", "<f8"), ("after", "<f8"), ("cls", "<i4"),
                   ("kind", "<i4")])
CAP = 96  # fix records per trial (36 tiles; MUST needs 1 each)
TDT = {"f64": torch.float64, "f32": torch.float32}
NDT = {"f64": np.float64, "f32": np.float32}
IDT = {"f64": torch.int64, "f32": torch.int32}
BITS = {"f64": 64, "f32": 32}
VAL_TOL = {"f64": 1e-12, "f32": 1e-5}


def _tiles():
    return [(I, J) for J in range(NT) for I in range(J, NT)]


def _positions(i, j):
    """(tile index, gi, gj) of the trial's flips: local (i, j) in every lower
    tile; diagonal tiles only when (i, j) is stored (i >= j)."""
    out = []
    for t, (I, J) in enumerate(_tiles()):
        if I == J and i < j:
            continue
        out.append((t, I * NB + i, J * NB + j))
    return out


def _flip(vals, bit, prec):
    a = np.asarray(vals, dtype=NDT[prec]).copy()
    u = a.view(np.uint64 if prec == "f64" else np.uint32)
    u ^= (np.uint64(1) << np.uint64(bit)) if prec == "f64" else (np.uint32(1) << np.uint32(bit))
    return u.view(NDT[prec]).astype(np.float64)


def _taus(st, gi, gj):
    """tau_e of every checksum vector the flip at stored (gi, gj) touches."""
    g = 2.0 * ck.gamma(NB, ck.unit_roundoff(st.prec))
    I, J = gi // NB, gj // NB
    t = [g * st.colmag[I, gj], g * st.rowmag[gi, J]]
    if I == J and gi != gj:  # the symmetric view sees the element twice
        i, j = gi - I * NB, gj - J * NB
        t += [g * st.colmag[I, J * NB + i], g * st.rowmag[I * NB + j, J]]
    return min(t), max(t)


def _band(delta, tmin, tmax):
    if not np.isfinite(delta) or abs(delta) >= 16 * NB * tmax:
        return "MUST"
    if abs(delta) <= tmin / 8:
        return "NEED_NOT"
    return "GRAY"


@pytest.mark.parametrize("prec", ["f64", "f32"])
def test_exhaustive_single_flip_campaign_config1(lib, prec):
    A_np = si.spd(N, seed=0).astype(NDT[prec]).astype(np.float64)
    st = ck.State.alloc(A_np, NB, prec=prec)
    ck.encode(st, ck.Tiles(0, NT, 0, NT, True, ck.SYM_LOWER))

    A = dev(A_np, TDT[prec])
    mat = lib.Mat.alloc(A, NB)
    t = lib.tiles(0, NT, 0, NT, True, lib.SYM_LOWER)
    lib.abft_encode(mat, t)
    clean = [x.clone() for x in (mat.A, mat.colchk, mat.rowchk, mat.colmag, mat.rowmag)]
    tol = lib.abft_tol_t(lib.TOL_MAGNITUDE, 1.0)
    Aint = mat.A.view(IDT[prec])

    combos = [(i, j, b) for i in range(NB) for j in range(NB) for b in range(BITS[prec])]
    T = len(combos)
    ntile = len(_tiles())
    status_v = torch.zeros((T, NT, NT), dtype=torch.int32, device="cuda")
    status_all = torch.zeros((T, NT, NT), dtype=torch.int32, device="cuda")
    counts_all = torch.zeros((T, 8), dtype=torch.int32, device="cuda")
    nfix_all = torch.zeros(T, dtype=torch.int32, device="cuda")
    fix_all = torch.zeros((T, CAP * lib.FIX_BYTES), dtype=torch.uint8, device="cuda")
    vals_all = torch.zeros((T, ntile), dtype=torch.float64, device="cuda")
    other_all = torch.zeros((T, NT, NT), dtype=torch.int32, device="cuda")
    pos_cache = {}
    for tr, (i, j, b) in enumerate(combos):
        if (i, j) not in pos_cache:
            pos = _positions(i, j)
            ti = torch.tensor([p[0] for p in pos], device="cuda")
            gi = torch.tensor([p[1] for p in pos], device="cuda")
            gj = torch.tensor([p[2] for p in pos], device="cuda")
            keep = torch.ones((N, N), dtype=torch.bool, device="cuda")
            keep[gi, gj] = False
            pos_cache[(i, j)] = (ti, gi, gj, keep)
        ti, gi, gj, keep = pos_cache[(i, j)]
        for dst, src in zip((mat.A, mat.colchk, mat.rowchk, mat.colmag, mat.rowmag), clean):
            dst.copy_(src)
        mask = (1 << b) if b < BITS[prec] - 1 else -(1 << (BITS[prec] - 1))  # sign bit as a signed int
        Aint[gi, gj] = Aint[gi, gj] ^ mask
        rep = lib.Report(status_all[tr].t(), counts_all[tr])
        lib.abft_verify(mat, t, lib.BOTH, tol, rep)
        status_v[tr].copy_(status_all[tr])
        lib.abft_locate_correct(mat, t, lib.BOTH, tol, rep, fix_all[tr], nfix_all[tr:tr + 1])
        vals_all[tr, ti] = mat.A[gi, gj].double()
        # elements other than the flipped ones that the locate step changed, per tile (I, J)
        other_all[tr] = ((mat.A != clean[0]) & keep).reshape(NT, NB, NT, NB).sum((1, 3))
    torch.cuda.synchronize()

    sv, sf = status_v.cpu().numpy(), status_all.cpu().numpy()  # [trial, J, I] (column-major status)
    nf, vals, other = nfix_all.cpu().numpy(), vals_all.cpu().numpy(), other_all.cpu().numpy()  # other: [trial, I, J]
    fixes = fix_all.cpu().numpy()
    # per (i, j): the flipped positions and their thresholds (error-free state)
    meta = {}
    for (i, j) in pos_cache:
        pos = _positions(i, j)
        ti = np.array([p[0] for p in pos])
        gi = np.array([p[1] for p in pos])
        gj = np.array([p[2] for p in pos])
        tt = np.array([_taus(st, a, c) for a, c in zip(gi, gj)])
        meta[(i, j)] = (ti, gi, gj, gi // NB, gj // NB, A_np[gi, gj], tt[:, 0], tt[:, 1])
    tally = {"MUST": 0, "NEED_NOT": 0, "GRAY": 0}
    gray_out = {"fixed": 0, "undetected": 0, "uncorrectable": 0, "other": 0}
    must_by_bit = np.zeros(BITS[prec], dtype=np.int64)
    fails = []
    g = si.rng(11)
    sample_tr = set()
    for b in range(BITS[prec]):
        for _ in range(4):
            i, j = int(g.integers(0, NB)), int(g.integers(0, NB))
            sample_tr.add((i * NB + j) * BITS[prec] + b)
    for tr, (i, j, b) in enumerate(combos):
        assert nf[tr] <= CAP
        ti, gi, gj, I, J, x0, tmin, tmax = meta[(i, j)]
        xf = _flip(x0, b, prec)
        with np.errstate(invalid="ignore", over="ignore"):
            delta = np.where(np.isfinite(xf), xf - x0, np.inf)
            must = ~np.isfinite(delta) | (np.abs(delta) >= 16 * NB * tmax)
            neednot = ~must & (np.abs(delta) <= tmin / 8)
        gray = ~must & ~neednot
        tally["MUST"] += int(must.sum())
        tally["NEED_NOT"] += int(neednot.sum())
        tally["GRAY"] += int(gray.sum())
        must_by_bit[b] += int(must.sum())
        recs = np.frombuffer(fixes[tr, :nf[tr] * FIX_DT.itemsize].tobytes(), dtype=FIX_DT)
        rt = (recs["gi"] // NB) * NT + recs["gj"] // NB  # tile of each record
        tid = I * NT + J
        nrec = np.bincount(rt, minlength=NT * NT)[tid]
        flagged = sv[tr, J, I] != 0
        clean_after = sf[tr, J, I] == 0
        oth = other[tr, I, J]
        v = vals[tr, ti]
        first = {}
        for r in recs:
            first.setdefault(int(r["gi"] // NB) * NT + int(r["gj"] // NB), r)
        for k in np.nonzero(must)[0]:
            r = first.get(int(tid[k]))
            ok = (flagged[k] and clean_after[k] and nrec[k] == 1 and oth[k] == 0 and r is not None
                  and r["gi"] == gi[k] and r["gj"] == gj[k] and r["cls"] == ck.CLS_0D and r["kind"] == ck.FIX_DATA
                  and abs(v[k] - x0[k]) <= tmin[k])
            if not ok:
                fails.append(("MUST", i, j, b, int(I[k]), int(J[k]), int(sv[tr, J[k], I[k]]), int(sf[tr, J[k], I[k]]),
                              None if r is None else r.tolist(), float(v[k]), float(x0[k])))
        for k in np.nonzero(neednot)[0]:
            if flagged[k] or nrec[k] or oth[k] or v[k] != xf[k]:
                fails.append(("NEED_NOT", i, j, b, int(I[k]), int(J[k]), int(sv[tr, J[k], I[k]])))
        for k in np.nonzero(gray)[0]:
            if not flagged[k]:
                gray_out["undetected"] += 1
            elif sf[tr, J[k], I[k]] & ck.ST_UNCORRECTABLE:
                gray_out["uncorrectable"] += 1
            elif abs(v[k] - x0[k]) <= tmin[k] and oth[k] == 0:
                gray_out["fixed"] += 1
            else:
                gray_out["other"] += 1
    summary = {"prec": prec, "n": N, "nb": NB, "trials": T, "flips": int(sum(tally.values())), "bands": tally,
               "gray_outcomes": gray_out, "must_by_bit": must_by_bit.tolist(), "must_failures": len(fails)}
    out = os.path.join(os.environ.get("GRAFT_REPO_ROOT", "."), "gpurun_out")
    if os.path.isdir(out):
        with open(os.path.join(out, f"flip_campaign_config1_{prec}.json"), "w") as f:
            json.dump(summary, f, indent=1)
    print(json.dumps(summary))
    assert not fails, fails[:10]
    assert tally["MUST"] > 0 and tally["NEED_NOT"] > 0

    # ---- oracle parity on the stratified sample --------------------------
    for tr in sorted(sample_tr):
        i, j, b = combos[tr]
        so = st.copy()
        for ti, gi, gj in _positions(i, j):
            so.A[gi, gj] = float(_flip([A_np[gi, gj]], b, prec)[0])
        tt = ck.Tiles(0, NT, 0, NT, True, ck.SYM_LOWER)
        osv, _ = ck.verify(so, tt, ck.BOTH)
        osf, ofix, _ = ck.locate_correct(so, tt, ck.BOTH)
        recs = np.frombuffer(fixes[tr, :nf[tr] * FIX_DT.itemsize].tobytes(), dtype=FIX_DT)
        for ti, gi, gj in _positions(i, j):
            I, J = gi // NB, gj // NB
            x0 = A_np[gi, gj]
            xf = float(_flip([x0], b, prec)[0])
            delta = xf - x0 if np.isfinite(xf) else np.inf
            if _band(delta, *_taus(st, gi, gj)) == "GRAY":
                continue
            # fp32: ST_NONFINITE records an fp32 overflow of the recomputed
            # sums (a bit-30 flip makes ~1e38); the oracle sums fp32 data in
            # fp64 (c-21), so only the flag bits are compared there
            nfm = ~ck.ST_NONFINITE if prec == "f32" else -1
            assert sv[tr, J, I] & nfm == osv[(I, J)] & nfm, (tr, I, J, sv[tr, J, I], osv[(I, J)])
            assert sf[tr, J, I] == osf[(I, J)], (tr, I, J)
            mine = sorted((int(r["gi"]), int(r["gj"]), int(r["cls"]), int(r["kind"]))
                          for r in recs if r["gi"] // NB == I and r["gj"] // NB == J)
            theirs = sorted((f.gi, f.gj, f.cls, f.kind) for f in ofix if f.gi // NB == I and f.gj // NB == J)
            assert mine == theirs, (tr, I, J, mine, theirs)
            if np.isfinite(so.A[gi, gj]):
                assert abs(vals[tr, ti] - so.A[gi, gj]) <= VAL_TOL[prec] * np.abs(A_np).max(), (tr, I, J)
