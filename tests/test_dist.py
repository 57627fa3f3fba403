"""Host logic of the distributed driver (row e) that mgpu.ft_potrf_mgpu
calls: block-cyclic layout, the broadcast groups (which ranks need which
panel piece), the L361-L363 decision, and — with world_size 2 over gloo on
CPU — the groups' creation, a group broadcast and the decision exchange."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_chenlllwtolzgc18_b200 import dist as D


def test_grid_shapes():
    assert [D.grid_shape(w) for w in (1, 2, 4, 8)] == [(1, 1), (1, 2), (2, 2), (2, 4)]


@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_block_cyclic_partition(world):
    P, Q = D.grid_shape(world)
    n, nb = 12 * 4, 4
    seen = {}
    for r in range(world):
        L = D.Layout(n, nb, P, Q, r)
        for t in L.tiles():
            assert t not in seen
            seen[t] = r
            assert L.owner(*t) == r
    assert len(seen) == (n // nb) ** 2
    low = [t for r in range(world) for t in D.Layout(n, nb, P, Q, r).tiles(lower_only=True)]
    assert sorted(low) == sorted((I, J) for J in range(n // nb) for I in range(J, n // nb))


@pytest.mark.parametrize("P,Q", [(1, 1), (1, 2), (2, 1), (2, 2), (2, 4), (1, 3), (3, 2), (2, 3), (4, 2)])
def test_piece_groups_hold_every_rank_that_needs_the_piece(P, Q):
    """Brute force over every iteration: a rank that uses panel piece pp —
    as its row operand (its process row) or for one of its tile columns J
    (lcol_sources) — is in piece_ranks(pp); the sender (pp, k mod Q) too;
    the diagonal tile's receivers (the panel owners) form column_ranks."""
    n, nb = 13 * 4, 4
    nt = n // nb
    for k in range(nt - 1):
        kq = k % Q
        for r in range(P * Q):
            L = D.Layout(n, nb, P, Q, r)
            need = {L.p} if L.piece_count(k, L.p) else set()
            need |= {pp for pp, _ in L.lcol_sources(k)}
            for pp in need:
                assert r in D.piece_ranks(P, Q, pp), (k, r, pp)
        for pp in range(P):
            assert pp * Q + kq in D.piece_ranks(P, Q, pp)
        assert sorted(D.column_ranks(P, Q, kq)) == sorted(r for r in range(P * Q) if r % Q == kq)
    # 2 x 4: each piece reaches 6 of the 8 ranks (not the whole world)
    if (P, Q) == (2, 4):
        assert [len(D.piece_ranks(P, Q, pp)) for pp in range(P)] == [6, 6]


def test_classify_bcast():
    assert D.classify_bcast(0, 3) == "clean"
    assert D.classify_bcast(1, 3) == "communication"
    assert D.classify_bcast(3, 3) == "restart"
    assert D.classify_bcast(0, 3, sender_2d=1) == "restart"  # the sender's own check left a 2D error
    assert D.classify_bcast(1, 1) == "restart"  # a single receiver cannot tell (L363: "all GPUs")
    assert D.classify_bcast(0, 0) == "clean"


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        P, Q = D.grid_shape(world)
        G = D.Groups(P, Q)  # collective: every rank creates every group
        # a piece broadcast inside its group (mgpu's round), sender = rank 1
        buf = torch.full((4,), float(rank))
        if rank in G.piece_ranks[0]:
            dist.broadcast(buf, src=1, group=G.piece[0])
        # decision words: sender (rank 1) reports no 2D error, receiver flags
        w_all = torch.tensor([0, 1 if rank == 0 else 0], dtype=torch.int32)
        w_none = torch.tensor([0, 0], dtype=torch.int32)
        w_2d = torch.tensor([1 if rank == 1 else 0, 0], dtype=torch.int32)
        res = D.decide([(G.piece[0], w_all), (G.piece[0], w_none), (G.piece[0], w_2d)], world)
        counts = torch.tensor([rank + 1, 0, 2 * rank, 0, 0, 0, 0, rank], dtype=torch.int32)
        D.reduce_counts(counts)
        q.put((rank, buf.tolist(), res, counts.tolist(), G.piece_ranks, G.col_ranks))
    finally:
        dist.destroy_process_group()


def test_two_rank_groups_broadcast_and_decision():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, buf, dec, counts, pieces, cols in res:
        assert pieces == [[0, 1]] and cols == [[0], [1]]  # 1 x 2 grid
        assert buf == [1.0] * 4  # rank 1's piece reached rank 0
        # one receiver (rank 0) of rank 1's piece: it flagged -> "restart" (all
        # receivers); nobody -> clean; the sender's 2D -> restart
        assert dec == [[0, 1], [0, 0], [1, 0]]
        assert [D.classify_bcast(nf, 1, s2) for s2, nf in dec] == ["restart", "clean", "restart"]
        assert counts == [3, 0, 2, 0, 0, 0, 0, 1]
