"""Multi-GPU fault-tolerant Cholesky over a 2D block-cyclic tile grid
(SURVEY §8 row e; paper §VII.C).

One process per GPU.  Tile (I, J) of the n x n matrix (nb x nb tiles) lives
on rank (I mod P) * Q + (J mod Q) of a P x Q grid (`dist.grid_shape`); each
rank stores its tiles as one column-major local matrix with the checksum
state of `abft.Mat` (tile-local weights, so a local tile's checksums are the
global tile's).  Iteration k of Alg. 2 (L368-L378):

  1. owner of A_kk: pre-PD check (SYM_LOWER, c and r), PD + c(L_kk) rule
     (`abft_panel_potrf`), post-PD check (LOWER, c);
  2. diagonal round: L_kk | c(L_kk) | m_c(L_kk) is broadcast inside process
     column k mod Q (the panel owners, `dist.Groups.col`); every receiver
     verifies and corrects its copy (communication errors, L355), then the
     owner's post-PD verdict and the receivers' flags are all-reduced in the
     group and decided by L361-L363 (`dist.classify_bcast`): all receivers
     flagged, or the owner's check left a 2D error -> the owner restores its
     pre-PD copy, redoes the PD (L430) and broadcasts again; some -> the
     receivers' local corrections stand (communication error);
  3. panel owners: pre-PU check (c and r), PU L_ik = A_ik L_kk^-T and
     c(L_ik) = c(A_ik) L_kk^-T (`abft_update_trsm_inv`), post-PU check (c);
  4. piece rounds: each process row's panel piece goes (async, all pieces at
     once) to the ranks that need it (`dist.Groups.piece`: its process row
     and the process columns holding its tile columns), is checked by every
     receiver and decided as in 2 (restart -> the sender redoes its PU and
     broadcasts the piece again);
  5. every rank updates its local trailing tiles A_IJ -= L_ik L_jk^T with
     c(A_IJ) -= c(L_ik) L_jk^T and r(A_IJ) -= L_ik c(L_jk)^T (+ magnitudes,
     c-6, c-12), grouped tile columns per call (`abft_update_gemm`);
  6. the received panel is re-checked after the trailing update (Fig. 4a);
     a value corrected there was already consumed by the update, which the
     distributed driver reports as uncorrectable (no distributed repair,
     DESIGN §7 e-2); the panel owners re-check their stored pieces too.

Host synchronisation: one read of the all-reduced decision words per round
(2 per iteration; the decision is control flow), none for data movement (the
column-role index tensors are built once before the loop).  Only panels,
checksums and int32 error reports cross the interconnect; torch.distributed
is plumbing (NCCL on the GPU box; gloo with CUDA tensors when several ranks
share one GPU in the tests).  Every arithmetic step is a C-ABI call into
libabft_b200.so; the buffer packing below only moves bytes.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import torch
import torch.distributed as dist

from . import abft
from .dist import Groups, Layout, classify_bcast, grid_shape  # noqa: F401  (re-exported)
from .dist import decide as decide_round

AT_BCAST = 8   # fault hook: a receiver's copy of a broadcast panel (communication error)
AT_SEND = 11   # fault hook: the sender's packed buffer right before its first broadcast


def scatter_tiles(A: torch.Tensor, lay: Layout, device="cuda") -> torch.Tensor:
    """This rank's tiles of the global column-major matrix A (any device) as
    a local column-major matrix on `device` (plumbing: a copy)."""
    nb = lay.nb
    rows = torch.cat([torch.arange(I * nb, (I + 1) * nb) for I in range(lay.p, lay.nt, lay.P)]) \
        if lay.mt_loc else torch.zeros(0, dtype=torch.long)
    cols = torch.cat([torch.arange(J * nb, (J + 1) * nb) for J in range(lay.q, lay.nt, lay.Q)]) \
        if lay.nt_loc else torch.zeros(0, dtype=torch.long)
    blk = A.index_select(0, rows.to(A.device)).index_select(1, cols.to(A.device))
    return abft.to_colmajor(blk.to(device))


def gather_tiles(A_loc: torch.Tensor, lay: Layout, group=None) -> torch.Tensor:
    """Inverse of scatter_tiles, assembled on every rank (host tensor)."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    parts = [None] * world
    if world > 1:
        dist.all_gather_object(parts, A_loc.cpu(), group=group)
    else:
        parts = [A_loc.cpu()]
    n, nb = lay.n, lay.nb
    out = torch.zeros(n, n, dtype=A_loc.dtype)
    for r, blk in enumerate(parts):
        L = Layout(n, nb, lay.P, lay.Q, r)
        for il, I in enumerate(range(L.p, L.nt, L.P)):
            for jl, J in enumerate(range(L.q, L.nt, L.Q)):
                out[I * nb:(I + 1) * nb, J * nb:(J + 1) * nb] = blk[il * nb:(il + 1) * nb, jl * nb:(jl + 1) * nb]
    return out


class _Piece:
    """Broadcast buffer of cnt panel tiles: L (cnt*nb x nb) | c (2cnt x nb) |
    m_c (cnt x nb), all column-major, in one flat tensor."""

    def __init__(self, cnt, nb, dtype, device):
        self.cnt, self.nb = cnt, nb
        self.flat = torch.empty(cnt * nb * nb + 3 * cnt * nb, dtype=dtype, device=device)
        o1 = cnt * nb * nb
        o2 = o1 + 2 * cnt * nb
        self.Lu = self.flat[:o1].view(nb, cnt, nb)  # [col][tile][row]
        self.cu = self.flat[o1:o2].view(nb, cnt, 2)
        self.mu = self.flat[o2:].view(nb, cnt)

    @property
    def L(self):
        return self.Lu.reshape(self.nb, self.cnt * self.nb).t()

    @property
    def c(self):
        return self.cu.reshape(self.nb, 2 * self.cnt).t()

    @property
    def m(self):
        return self.mu.t()

    def mat(self):
        return abft.Mat(self.L, self.nb, self.c, None, self.m, None)


@dataclass
class MgpuStats:
    counts: list = field(default_factory=lambda: [0] * abft.NCOUNTS)
    bcast_counts: list = field(default_factory=lambda: [0] * abft.NCOUNTS)
    bcast_events: list = field(default_factory=list)  # (k, source, nflag, nrecv, kind)
    tmu_consumed: int = 0
    info: int = 0
    uncorrectable: int = 0
    restarts: int = 0


def ft_potrf_mgpu(A_loc: torch.Tensor, lay: Layout, abft_on=True, tol_scale=1.0, inject=(), group=None,
                  tmu_groups=32, restart=True, groups: Groups = None):
    """Fault-tolerant lower Cholesky of the distributed matrix in place.
    A_loc: this rank's local column-major matrix (from scatter_tiles).
    inject: (iter, point, gi, gj, xor_mask[, rank]) with global (gi, gj);
    point in abft.AT_* (applied by the tile's owner), AT_BCAST (applied to
    `rank`'s received copy of panel element (gi, gj) of iteration iter) or
    AT_SEND (applied by the sender to its packed buffer before the first
    broadcast: every receiver sees it).  groups: the broadcast communicators
    (dist.Groups; built here when None — a collective call on every rank).
    Returns (rc, MgpuStats); rc is 0 or abft.E_UNCORRECTABLE."""
    nb, nt, P, Q = lay.nb, lay.nt, lay.P, lay.Q
    p, q = lay.p, lay.q
    dev, dt = A_loc.device, A_loc.dtype
    world = P * Q
    me = lay.rank
    G = groups if groups is not None else Groups(P, Q, group)
    UNC = abft.NCOUNTS - 1
    tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, tol_scale, 1)
    mat = abft.Mat.alloc(A_loc, nb) if abft_on else abft.Mat(A_loc, nb)
    rep = abft.Report.alloc(mat) if abft_on else None
    rep_b = abft.Report(abft.colmajor_zeros(max(nt, 1), 1, dtype=torch.int32, device=dev),
                        torch.zeros(abft.NCOUNTS, dtype=torch.int32, device=dev))
    cb_total = torch.zeros(abft.NCOUNTS, dtype=torch.int32, device=dev)
    bflag = torch.zeros(nt, P + 1, dtype=torch.int32, device=dev)     # [k][piece | diag]: receivers that flagged
    brestart = torch.zeros(nt, P + 1, dtype=torch.int32, device=dev)  # [k][piece | diag]: restart + re-broadcast
    consumed = torch.zeros(1, dtype=torch.int32, device=dev)
    fixes = torch.zeros(4096 * abft.FIX_BYTES, dtype=torch.uint8, device=dev)
    nfix = torch.zeros(1, dtype=torch.int32, device=dev)
    infos = torch.zeros(max(nt, 1), dtype=torch.int32, device=dev)
    Linv = abft.colmajor_zeros(nb, nb, dtype=dt, device=dev)
    diag_buf = _Piece(1, nb, dt, dev)
    zero1 = torch.zeros(1, dtype=torch.int32, device=dev)
    sent = set()  # AT_SEND faults already applied (first send only)

    # the column-role sources of every iteration, as device index tensors,
    # built once (no host-to-device copies inside the loop)
    lcol_idx = []
    for k in range(nt):
        srcs = lay.lcol_sources(k)
        per = []
        for pp in range(P):
            sel = [t for t, (s_, _) in enumerate(srcs) if s_ == pp]
            if sel:
                per.append((pp, torch.tensor(sel, device=dev), torch.tensor([srcs[t][1] for t in sel], device=dev)))
        lcol_idx.append((len(srcs), per))

    def check(m, tl, which):
        abft.abft_check(m, tl, which, tol, rep, fixes, nfix)  # verify + fused locate, one launch

    def check_recv(m, tl, acc):
        """Post-broadcast check of a received copy (L355) into the round's
        counters `acc` (added to the run's totals once the round is decided)."""
        abft.abft_check(m, tl, abft.COL, tol, rep_b, fixes, nfix)
        acc.add_(rep_b.counts)
        rep_b.counts.zero_()

    def hook(k, point):
        for f in inject:
            it, pt, gi, gj, mask = f[:5]
            if it != k or pt != point or pt in (AT_BCAST, AT_SEND):
                continue
            if lay.owner(gi // nb, gj // nb) == me:
                li, lj = lay.to_local(gi, gj)
                abft.abft_inject(A_loc, li, lj, mask)

    def hook_buf(k, point, buf: _Piece, tiles_I):
        """A flip in a broadcast buffer: AT_BCAST in `rank`'s received copy,
        AT_SEND in the sender's packed buffer (first send only)."""
        for idx, f in enumerate(inject):
            it, pt, gi, gj, mask = f[:5]
            rk = f[5] if len(f) > 5 else -1
            if it != k or pt != point or gj // nb != k or gi // nb not in tiles_I:
                continue
            if point == AT_BCAST and rk != me:
                continue
            if point == AT_SEND:
                if idx in sent:
                    continue
                sent.add(idx)
            t = tiles_I.index(gi // nb)
            abft.abft_inject(buf.L, t * nb + gi % nb, gj % nb, mask)

    restarts = [0]
    rs = abft_on and restart

    def snapshot(*ts):
        return [t.clone() for t in ts] + [rep.counts[UNC].clone()]

    def restore(snap, *ts):
        for t, c in zip(ts, snap[:-1]):
            t.copy_(c)
        rep.counts[UNC] = snap[-1]
        restarts[0] += 1

    def sub(m: abft.Mat, il, jl):
        """One local tile as its own 1x1-tile Mat (views into m's arrays)."""
        r0, c0 = il * nb, jl * nb
        return abft.Mat(m.A[r0:r0 + nb, c0:c0 + nb], nb,
                        m.colchk[2 * il:2 * il + 2, c0:c0 + nb] if m.colchk is not None else None,
                        m.rowchk[r0:r0 + nb, 2 * jl:2 * jl + 2] if m.rowchk is not None else None,
                        m.colmag[il:il + 1, c0:c0 + nb] if m.colmag is not None else None,
                        m.rowmag[r0:r0 + nb, jl:jl + 1] if m.rowmag is not None else None)

    def pack(buf: _Piece, A_view, c_view, m_view):
        buf.L.copy_(A_view)
        if abft_on:
            buf.c.copy_(c_view)
            buf.m.copy_(m_view)

    def decide(pairs):
        return decide_round(pairs, world)

    # ---- encode: the lower tiles of every local tile column (diag in SYM view)
    if abft_on:
        for jl in range(lay.nt_loc):
            J = jl * Q + q
            i0 = lay.row_first(J)
            if i0 < lay.mt_loc and i0 * P + p == J:
                abft.abft_encode(sub(mat, i0, jl), abft.tiles(0, 1, 0, 1, False, abft.SYM_LOWER))
                i0 += 1
            if i0 < lay.mt_loc:
                abft.abft_encode(mat, abft.tiles(i0, lay.mt_loc, jl, jl + 1))

    for k in range(nt):
        kp, kq = k % P, k % Q
        owner_kk = kp * Q + kq
        ik, jk = k // P, k // Q
        in_col = q == kq
        # ---- 1. PD on the owner of A_kk
        if me == owner_kk:
            D = sub(mat, ik, jk)
            hook(k, abft.AT_PRE_PD_CHECK)
            if abft_on:
                check(D, abft.tiles(0, 1, 0, 1, False, abft.SYM_LOWER), abft.BOTH)
            if rs:
                pd_snap = snapshot(D.A, D.colchk, D.colmag)

            def pd():
                abft.abft_panel_potrf(D, infos[k:k + 1], Linv)
                if abft_on:
                    check(D, abft.tiles(0, 1, 0, 1, False, abft.LOWER), abft.COL)

            hook(k, abft.AT_PRE_PD)
            if abft_on:
                unc0 = rep.counts[UNC].clone()
            abft.abft_panel_potrf(D, infos[k:k + 1], Linv)
            hook(k, abft.AT_POST_PD)
            if abft_on:
                check(D, abft.tiles(0, 1, 0, 1, False, abft.LOWER), abft.COL)
            pack(diag_buf, D.A, D.colchk, D.colmag)
            hook_buf(k, AT_SEND, diag_buf, [k])
        # ---- 2. diagonal round inside process column k mod Q
        if in_col:
            for attempt in range(2):
                if P > 1:
                    dist.broadcast(diag_buf.flat, src=owner_kk, group=G.col[kq])
                acc = torch.zeros(abft.NCOUNTS, dtype=torch.int32, device=dev)
                if me != owner_kk:
                    if attempt == 0:
                        hook_buf(k, AT_BCAST, diag_buf, [k])
                    if abft_on:
                        check_recv(diag_buf.mat(), abft.tiles(0, 1, 0, 1, False, abft.LOWER), acc)
                if not abft_on:
                    break
                word = torch.zeros(2, dtype=torch.int32, device=dev)
                if me == owner_kk:
                    word[0:1] = rep.counts[UNC:UNC + 1] - unc0
                else:
                    word[1:2] = (acc[0:1] > 0).to(torch.int32)
                if attempt == 0 and me != owner_kk:
                    bflag[k, P] += word[1]
                s2d, nflag = decide([(G.col[kq], word)])[0]
                if attempt == 1 or classify_bcast(nflag, P - 1, s2d) != "restart" or not rs:
                    cb_total.add_(acc)
                    break
                # L363 / L430: restart of the PD on the owner, broadcast again
                if me == owner_kk:
                    restore(pd_snap, D.A, D.colchk, D.colmag)
                    brestart[k, P] += 1
                    unc0 = rep.counts[UNC].clone()
                    pd()
                    pack(diag_buf, D.A, D.colchk, D.colmag)
            if me != owner_kk:
                abft.abft_tri_inverse("L", "N", diag_buf.L, Linv)
        if k == nt - 1:
            break
        # ---- 3. PU on the panel owners
        ir0 = lay.row_first(k + 1)
        cnt = lay.mt_loc - ir0
        pan = None
        if in_col and cnt > 0:
            r0 = ir0 * nb
            hook(k, abft.AT_PRE_PU_CHECK)
            if abft_on:
                check(mat, abft.tiles(ir0, lay.mt_loc, jk, jk + 1), abft.BOTH)
            pan = (A_loc[r0:, jk * nb:(jk + 1) * nb],) + ((mat.colchk[2 * ir0:, jk * nb:(jk + 1) * nb],
                                                            mat.colmag[ir0:, jk * nb:(jk + 1) * nb]) if abft_on else ())
            if rs:
                pu_snap = snapshot(*pan)

            def pu():
                abft.abft_update_trsm_inv("R", "T", Linv, pan[0], cnt * nb)
                if abft_on:
                    abft.abft_update_trsm_inv("R", "T", Linv, pan[1], 2 * cnt, pan[2], cnt)

            hook(k, abft.AT_PRE_PU)
            if abft_on:
                unc_pu = rep.counts[UNC].clone()
            pu()
            hook(k, abft.AT_POST_PU)
            if abft_on:
                check(mat, abft.tiles(ir0, lay.mt_loc, jk, jk + 1), abft.COL)
        # ---- 4. piece rounds: each piece to the ranks that need it
        pieces, tiles_of = [None] * P, [None] * P
        for pp in range(P):
            c_pp = lay.piece_count(k, pp)
            if c_pp and me in G.piece_ranks[pp]:
                pieces[pp] = _Piece(c_pp, nb, dt, dev)
                first = lay.row_first(k + 1, pp)
                tiles_of[pp] = [(first + t) * P + pp for t in range(c_pp)]
        sender = [pp * Q + kq for pp in range(P)]
        if pan is not None:
            pack(pieces[p], pan[0], pan[1] if abft_on else None, pan[2] if abft_on else None)
            hook_buf(k, AT_SEND, pieces[p], tiles_of[p])

        def piece_round(pps, first):
            if world > 1:
                works = [dist.broadcast(pieces[pp].flat, src=sender[pp], group=G.piece[pp], async_op=True)
                         for pp in pps]
                for w in works:
                    w.wait()
            accs = {}
            for pp in pps:
                accs[pp] = torch.zeros(abft.NCOUNTS, dtype=torch.int32, device=dev)
                if me != sender[pp]:
                    if first:
                        hook_buf(k, AT_BCAST, pieces[pp], tiles_of[pp])
                    if abft_on:
                        check_recv(pieces[pp].mat(), abft.tiles(0, pieces[pp].cnt, 0, 1), accs[pp])
            return accs

        live = [pp for pp in range(P) if pieces[pp] is not None]
        accs = piece_round(live, True)
        if abft_on and live:
            words = []
            for pp in live:
                w = torch.zeros(2, dtype=torch.int32, device=dev)
                if me == sender[pp]:
                    w[0:1] = rep.counts[UNC:UNC + 1] - unc_pu
                else:
                    w[1:2] = (accs[pp][0:1] > 0).to(torch.int32)
                    bflag[k, pp] += w[1]
                words.append((G.piece[pp], w))
            res = decide(words)
            redo = [pp for pp, (s2d, nflag) in zip(live, res)
                    if rs and classify_bcast(nflag, len(G.piece_ranks[pp]) - 1, s2d) == "restart"]
            for pp in live:
                if pp not in redo:
                    cb_total.add_(accs[pp])
            if redo:
                # L363 / L430: the sender restores its pre-PU copy, redoes the
                # PU (and its check) and the piece is broadcast again
                if p in redo and pan is not None:
                    restore(pu_snap, *pan)
                    brestart[k, p] += 1
                    pu()
                    check(mat, abft.tiles(ir0, lay.mt_loc, jk, jk + 1), abft.COL)
                    pack(pieces[p], pan[0], pan[1], pan[2])
                for pp, acc in piece_round(redo, False).items():
                    cb_total.add_(acc)
        # ---- 5. trailing update of the local tiles I >= J > k
        ncol, per = lcol_idx[k]
        Lrow = pieces[p]
        if ncol and Lrow is not None:
            Lcol = _Piece(ncol, nb, dt, dev)
            for pp, dst_idx, src_idx in per:
                Lcol.Lu.index_copy_(1, dst_idx, pieces[pp].Lu.index_select(1, src_idx))
                Lcol.cu.index_copy_(1, dst_idx, pieces[pp].cu.index_select(1, src_idx))
                Lcol.mu.index_copy_(1, dst_idx, pieces[pp].mu.index_select(1, src_idx))
            hook(k, abft.AT_PRE_TMU)
            jl0 = lay.col_first(k + 1)
            # data: tile-column groups, rows from the group's first diagonal
            # tile (the upper tiles inside a group are computed and unused:
            # <= 1/tmu_groups of the flops)
            g = max(1, math.ceil(ncol / max(1, tmu_groups)))
            for ta in range(0, ncol, g):
                tb = min(ncol, ta + g)
                ia = lay.row_first((jl0 + ta) * Q + q)
                rows = lay.mt_loc - ia
                if rows <= 0:
                    continue
                s0 = ia - ir0  # first Lrow tile used
                abft.abft_update_gemm(abft.COL, "N", "T", -1.0, Lrow.L[s0 * nb:, :], Lcol.L[ta * nb:tb * nb, :],
                                      A_loc[ia * nb:, (jl0 + ta) * nb:(jl0 + tb) * nb], rows * nb, (tb - ta) * nb, nb)
            if abft_on:
                # checksums of the whole local trailing block, one product per
                # side (entries of upper tiles are updated and never read):
                # c(A_IJ) -= c(L_ik) L_jk^T,  r(A_IJ) -= L_ik c(L_jk)^T  (c-12)
                abft.abft_update_gemm(abft.COL, "N", "T", -1.0, Lrow.c, Lcol.L, mat.colchk[2 * ir0:, jl0 * nb:],
                                      2 * cnt, ncol * nb, nb, Lrow.m, mat.colmag[ir0:, jl0 * nb:])
                abft.abft_update_gemm(abft.ROW, "T", "N", -1.0, Lcol.c, Lrow.L, mat.rowchk[ir0 * nb:, 2 * jl0:],
                                      2 * ncol, cnt * nb, nb, Lcol.m, mat.rowmag[ir0 * nb:, jl0:])
            hook(k, abft.AT_POST_TMU)
            # ---- 6. Fig. 4a re-check of the panel copies the update read
            if abft_on:
                before = nfix.clone()
                for buf in (Lrow, Lcol):
                    abft.abft_check(buf.mat(), abft.tiles(0, buf.cnt, 0, 1), abft.COL, tol, rep_b, fixes, nfix)
                consumed.add_(nfix - before)
                cb_total.add_(rep_b.counts)
                rep_b.counts.zero_()
        else:
            hook(k, abft.AT_PRE_TMU)
            hook(k, abft.AT_POST_TMU)
        # ---- 6b. the panel owners' stored pieces (the factor itself): Alg. 2
        # line 13 re-checks the panel after the TMU; here the update read the
        # broadcast copies (checked above), so a fault in the stored piece
        # since its post-PU check was consumed by nobody and is a plain fix
        if abft_on and in_col and cnt > 0:
            check(mat, abft.tiles(ir0, lay.mt_loc, jk, jk + 1), abft.COL)

    # ---- error reports: one all-reduce of the int32 counters (L361-L363)
    rep_counts = rep.counts if rep is not None else torch.zeros(abft.NCOUNTS, dtype=torch.int32, device=dev)
    nrs = torch.tensor([restarts[0]], dtype=torch.int32, device=dev)
    summary = torch.cat([rep_counts, cb_total, consumed, infos, bflag.reshape(-1), brestart.reshape(-1), nrs])
    if world > 1:
        dist.all_reduce(summary, op=dist.ReduceOp.SUM, group=group)
    h = summary.cpu().tolist()
    st = MgpuStats()
    st.counts = h[:8]
    st.bcast_counts = h[8:16]
    st.tmu_consumed = h[16]
    inf = h[17:17 + nt]
    nb_slots = nt * (P + 1)
    bf = h[17 + nt:17 + nt + nb_slots]
    br = h[17 + nt + nb_slots:17 + nt + 2 * nb_slots]
    st.restarts = h[-1]
    for kk in range(nt):
        if inf[kk] and not st.info:
            st.info = kk * nb + inf[kk]
        for slot in range(P + 1):
            nflag, nre = bf[kk * (P + 1) + slot], br[kk * (P + 1) + slot]
            if nflag or nre:
                nrecv = (P - 1) if slot == P else len(G.piece_ranks[slot]) - 1  # diag: the rest of process column k
                st.bcast_events.append((kk, slot, nflag, nrecv, classify_bcast(nflag, nrecv, nre)))
    st.uncorrectable = st.counts[abft.NCOUNTS - 1] + st.bcast_counts[abft.NCOUNTS - 1] + st.tmu_consumed
    rc = abft.E_UNCORRECTABLE if st.uncorrectable else 0
    return rc, st
