"""Host logic of the distributed driver (row e): block-cyclic maps, panel
pieces, the column-role sources and the L361-L363 classification."""
import itertools

import pytest
import torch

from paper_conf_sc_chenlllwtolzgc18_b200 import dist as D
from paper_conf_sc_chenlllwtolzgc18_b200 import mgpu


@pytest.mark.parametrize("P,Q", [(1, 1), (1, 2), (2, 1), (2, 2), (2, 4), (1, 3), (3, 2)])
def test_layout_partitions_tiles(P, Q):
    n, nb = 13 * 8, 8
    nt = n // nb
    seen = {}
    for r in range(P * Q):
        L = mgpu.Layout(n, nb, P, Q, r)
        assert (L.p, L.q) == divmod(r, Q)
        for I, J in L.tiles():
            assert L.owner(I, J) == r == (I % P) * Q + J % Q
            seen[(I, J)] = r
        assert L.mt_loc * L.nt_loc == len(L.tiles())
    assert len(seen) == nt * nt


@pytest.mark.parametrize("P,Q", [(1, 2), (2, 2), (2, 4), (3, 2)])
def test_pieces_and_sources(P, Q):
    n, nb = 11 * 4, 4
    nt = n // nb
    for k in range(nt - 1):
        # pieces cover the panel tiles I > k exactly once, in process-row order
        tiles = []
        for pp in range(P):
            L0 = mgpu.Layout(n, nb, P, Q, pp * Q)
            first = L0.row_first(k + 1, pp)
            c = L0.piece_count(k, pp)
            got = [(first + t) * P + pp for t in range(c)]
            assert all(I > k and I % P == pp for I in got)
            tiles += got
        assert sorted(tiles) == list(range(k + 1, nt))
        for r in range(P * Q):
            L = mgpu.Layout(n, nb, P, Q, r)
            js = [jl * Q + L.q for jl in range(L.col_first(k + 1), L.nt_loc)]
            assert all(J > k and J % Q == L.q for J in js)
            for J, (pp, idx) in zip(js, L.lcol_sources(k)):
                first = L.row_first(k + 1, pp)
                assert (first + idx) * P + pp == J


def test_first_at_least():
    for x, r, S in itertools.product(range(0, 20), range(0, 4), range(1, 5)):
        if r >= S:
            continue
        i = mgpu.Layout.first_at_least(x, r, S)
        assert i * S + r >= x and (i == 0 or (i - 1) * S + r < x)


@pytest.mark.parametrize("P,Q", [(1, 1), (2, 2), (1, 3)])
def test_scatter_gather_roundtrip(P, Q):
    n, nb = 48, 8
    A = torch.arange(n * n, dtype=torch.float64).reshape(n, n)
    parts = [mgpu.scatter_tiles(A, mgpu.Layout(n, nb, P, Q, r), device="cpu") for r in range(P * Q)]
    out = torch.zeros_like(A)
    for r, blk in enumerate(parts):
        L = mgpu.Layout(n, nb, P, Q, r)
        for il, I in enumerate(range(L.p, L.nt, L.P)):
            for jl, J in enumerate(range(L.q, L.nt, L.Q)):
                out[I * nb:(I + 1) * nb, J * nb:(J + 1) * nb] = blk[il * nb:(il + 1) * nb, jl * nb:(jl + 1) * nb]
    assert torch.equal(out, A)


def test_to_local():
    n, nb, P, Q = 64, 8, 2, 2
    for r in range(4):
        L = mgpu.Layout(n, nb, P, Q, r)
        for gi, gj in [(0, 0), (9, 17), (63, 40), (24, 55)]:
            if L.owner(gi // nb, gj // nb) != r:
                continue
            li, lj = L.to_local(gi, gj)
            assert (li // nb) * P + L.p == gi // nb and li % nb == gi % nb
            assert (lj // nb) * Q + L.q == gj // nb and lj % nb == gj % nb


def test_classify_bcast():
    assert mgpu.classify_bcast is D.classify_bcast
    assert mgpu.classify_bcast(0, 3) == "clean"
    assert mgpu.classify_bcast(1, 3) == "communication"
    assert mgpu.classify_bcast(3, 3) == "restart"
