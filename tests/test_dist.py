"""Multi-process (world_size 2, gloo, CPU) tests of the multi-GPU host logic:
block-cyclic ownership, the error-count all-reduce and the paper's
communication-vs-PD/PU error decision (L361–L363)."""
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
    mt = nt = 12
    seen = {}
    for r in range(world):
        for t in D.local_tiles(r, P, Q, mt, nt):
            assert t not in seen
            seen[t] = r
            assert D.owner(*t, P, Q) == r
    assert len(seen) == mt * nt
    # lower-only (Cholesky) partition covers exactly the lower tiles
    low = [t for r in range(world) for t in D.local_tiles(r, P, Q, mt, nt, lower_only=True)]
    assert sorted(low) == sorted((I, J) for J in range(nt) for I in range(J, mt))


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
        counts = torch.tensor([rank + 1, 0, 2 * rank, 0, 0, 0, 0, rank], dtype=torch.int32)
        D.reduce_counts(counts)
        all_bad = D.panel_error_kind(torch.tensor(1))
        one_bad = D.panel_error_kind(torch.tensor(1 if rank == 0 else 0))
        none = D.panel_error_kind(torch.tensor(0))
        q.put((rank, counts.tolist(), all_bad, one_bad, none))
    finally:
        dist.destroy_process_group()


def test_two_rank_error_exchange():
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
    for rank, counts, all_bad, one_bad, none in res:
        assert counts == [3, 0, 2, 0, 0, 0, 0, 1]
        assert all_bad == "restart" and one_bad == "communication" and none == "clean"
