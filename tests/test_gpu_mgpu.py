"""Row e: the distributed ft_potrf (2D block-cyclic, panel broadcasts,
post-broadcast checks) against the oracle's Cholesky.  Several ranks share
cuda:0 over gloo (NCCL refuses two ranks on one device), so the whole
multi-GPU algorithm runs on the single test GPU; the bench runs it over NCCL.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import synth_inputs as si
from oracle import updates as ou
from paper_conf_sc_chenlllwtolzgc18_b200 import abft, mgpu
from paper_conf_sc_chenlllwtolzgc18_b200 import dist as D

from . import mgpu_worker

pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(tmp_path, n, nb, grid, inject=(), abft_on=True, seed=11, restart=True):
    world = grid[0] * grid[1]
    out = str(tmp_path / f"mgpu_{grid[0]}x{grid[1]}.pt")
    mp.spawn(mgpu_worker.run, args=(world, _port(), n, nb, grid, list(inject), out, abft_on, seed, restart),
             nprocs=world, join=True)
    return torch.load(out)


def _ref(n, seed=11):
    Lref, info = ou.potrf_lower(si.spd(n, seed=seed))
    assert info == 0
    return Lref


@pytest.mark.parametrize("grid", [(1, 1), (1, 2), (2, 1), (2, 2), (1, 3)])
def test_error_free_matches_lapack(tmp_path, grid):
    n, nb = 768, 64
    r = _run(tmp_path, n, nb, grid)
    Lref = _ref(n)
    L = r["L"].numpy()
    assert r["rc"] == 0 and r["info"] == 0
    assert sum(r["counts"]) == 0 and sum(r["bcast_counts"]) == 0 and not r["bcast_events"]
    assert np.abs(L - Lref).max() <= 1e-12 * np.abs(Lref).max()


def test_unprotected_same_factor(tmp_path):
    n, nb = 512, 64
    r = _run(tmp_path, n, nb, (2, 2), abft_on=False)
    assert np.abs(r["L"].numpy() - _ref(n)).max() <= 1e-12 * np.abs(_ref(n)).max()


BIT = 1 << 61  # exponent bit: a MUST-band fault (reading c-10)


@pytest.mark.parametrize("case", [
    # (iter, point, gi, gj): global coordinates, n=512 nb=64
    (1, abft.AT_PRE_PD_CHECK, 100, 70),   # diag tile before its check
    (1, abft.AT_POST_PD, 110, 90),        # decomposed diag tile
    (0, abft.AT_PRE_PU_CHECK, 300, 20),   # panel before PU
    (2, abft.AT_POST_PU, 450, 140),       # updated panel
    (0, abft.AT_POST_TMU, 400, 200),      # trailing tile after the update (caught when it becomes panel)
    (1, abft.AT_PRE_TMU, 300, 70),        # owner's stored panel after its broadcast (Alg. 2 line 13)
    (2, abft.AT_POST_TMU, 470, 150),      # owner's stored panel after the update
])
def test_single_fault_corrected(tmp_path, case):
    n, nb = 512, 64
    it, pt, gi, gj = case
    r = _run(tmp_path, n, nb, (2, 2), inject=[(it, pt, gi, gj, BIT)])
    Lref = _ref(n)
    assert r["rc"] == 0, r
    assert r["counts"][0] >= 1 and r["counts"][5] >= 1  # a tile flagged, an element fixed
    assert np.abs(r["L"].numpy() - Lref).max() <= 1e-12 * np.abs(Lref).max()


@pytest.mark.parametrize("grid", [(2, 2), (1, 3)])
def test_communication_fault_one_receiver(tmp_path, grid):
    """A flip in one receiver's copy of the broadcast panel: detected and
    corrected by that receiver only -> 'communication' (L361-L363)."""
    n, nb = 512, 64
    world = grid[0] * grid[1]
    # iteration 1 panel element (row tile 5, column tile 1); pick a receiver that is not the sender
    k, gi, gj = 1, 5 * nb + 7, 1 * nb + 3
    pp = (gi // nb) % grid[0]
    sender = pp * grid[1] + (k % grid[1])
    members = D.piece_ranks(grid[0], grid[1], pp)  # the ranks that receive this piece
    recv = [r for r in members if r != sender][0]
    assert world >= len(members)
    r = _run(tmp_path, n, nb, grid, inject=[(k, mgpu.AT_BCAST, gi, gj, BIT, recv)])
    assert r["rc"] == 0, r
    assert r["bcast_counts"][5] >= 1  # an element fixed in a received copy
    kinds = [e[4] for e in r["bcast_events"]]
    assert kinds == ["communication"], r["bcast_events"]
    assert np.abs(r["L"].numpy() - _ref(n)).max() <= 1e-12 * np.abs(_ref(n)).max()


@pytest.mark.parametrize("grid", [(1, 1), (2, 2)])
def test_pd_consumed_fault_local_restart(tmp_path, grid):
    """A DRAM flip in A_kk between its pre-PD check and the PD is consumed by
    the PD (2D in L_kk): the owner restores its pre-PD copy and redoes the PD
    before the broadcast (f1, L430); without the restart it is uncorrectable."""
    n, nb = 512, 64
    inj = [(2, abft.AT_PRE_PD, 2 * nb + 40, 2 * nb + 9, BIT)]
    r0 = _run(tmp_path, n, nb, grid, inject=inj, restart=False)
    assert r0["rc"] == abft.E_UNCORRECTABLE
    r = _run(tmp_path, n, nb, grid, inject=inj)
    assert r["rc"] == 0 and r["restarts"] == 1, r
    assert np.abs(r["L"].numpy() - _ref(n)).max() <= 1e-12 * np.abs(_ref(n)).max()


@pytest.mark.parametrize("grid,what", [((1, 3), "piece"), ((2, 2), "diag"), ((2, 2), "piece")])
def test_all_receivers_flag_restart_and_rebroadcast(tmp_path, grid, what):
    """L361-L363 / L430: a flip in the SENDER's packed buffer reaches every
    receiver; all of them flag their copy, so the round decides 'restart':
    the sender redoes its PD / PU from its copy and broadcasts again; the
    receivers' first corrections are discarded and the factor is exact."""
    n, nb = 512, 64
    k = 1
    if what == "diag":
        gi, gj = k * nb + 20, k * nb + 5
    else:
        gi, gj = 6 * nb + 11, k * nb + 3
    r = _run(tmp_path, n, nb, grid, inject=[(k, mgpu.AT_SEND, gi, gj, BIT)])
    assert r["rc"] == 0, r
    assert r["restarts"] == 1, r
    kinds = [e[4] for e in r["bcast_events"]]
    assert kinds == ["restart"], r["bcast_events"]
    ev = r["bcast_events"][0]
    assert ev[2] == ev[3]  # every receiver flagged
    assert np.abs(r["L"].numpy() - _ref(n)).max() <= 1e-12 * np.abs(_ref(n)).max()
