"""Multi-GPU fault-tolerant Cholesky over a 2D block-cyclic tile grid
(SURVEY §8 row e; paper §VII.C).

One process per GPU.  Tile (I, J) of the n x n matrix (nb x nb tiles) lives
on rank (I mod P) * Q + (J mod Q) of a P x Q grid (`dist.grid_shape`); each
rank stores its tiles as one column-major local matrix with the checksum
state of `abft.Mat` (tile-local weights, so a local tile's checksums are the
global tile's).  Iteration k of Alg. 2 (L368-L378):

  1. owner of A_kk: pre-PD check (SYM_LOWER, c and r), PD + c(L_kk) rule
     (`abft_panel_potrf`), post-PD check (LOWER, c);
  2. broadcast L_kk | c(L_kk) | m_c(L_kk); receivers in process column k
     verify the received tile (communication errors, L355) and invert it;
  3. panel owners: pre-PU check (c and r), PU L_ik = A_ik L_kk^-T and
     c(L_ik) = c(A_ik) L_kk^-T (`abft_update_trsm_inv`), post-PU check (c);
  4. every panel piece (the tiles of one process row) is broadcast to all
     ranks, and every receiver verifies it against its column checksums and
     corrects it in place (L361-L363: all receivers flagged -> the sender's
     PD/PU was wrong; some -> communication error);
  5. every rank updates its local trailing tiles A_IJ -= L_ik L_jk^T with
     c(A_IJ) -= c(L_ik) L_jk^T and r(A_IJ) -= L_ik c(L_jk)^T (+ magnitudes,
     c-6, c-12), grouped tile columns per call (`abft_update_gemm`);
  6. the received panel is re-checked after the trailing update (Fig. 4a);
     a value corrected there was already consumed by the update, which the
     distributed driver reports as uncorrectable (no distributed repair);
     the panel owners re-check their stored pieces too (the factor itself,
     which no update read: a fault there is a plain fix).

Local restart (f1, L430): the owner of A_kk and the panel owners copy the
input of their PD / PU with its checksums after the pre-op check; a 2D error
left by their post-op check (read back on the host: one wait per op) restores
the copy and redoes the op once, before anything is broadcast.

Only panels, checksums and int32 error reports cross the interconnect;
torch.distributed is plumbing (NCCL on the GPU box; gloo with CUDA tensors
when several ranks share one GPU in the tests).  Every arithmetic step is a
C-ABI call into libabft_b200.so; the buffer packing below only moves bytes.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import torch
import torch.distributed as dist

from . import abft
from .dist import grid_shape

AT_BCAST = 8  # fault hook: a receiver's copy of the broadcast panel (communication error)


@dataclass
class Layout:
    """2D block-cyclic placement of nt x nt tiles on a P x Q grid."""

    n: int
    nb: int
    P: int
    Q: int
    rank: int

    @property
    def nt(self):
        return self.n // self.nb

    @property
    def p(self):
        return self.rank // self.Q

    @property
    def q(self):
        return self.rank % self.Q

    @property
    def mt_loc(self):
        return len(range(self.p, self.nt, self.P))

    @property
    def nt_loc(self):
        return len(range(self.q, self.nt, self.Q))

    def owner(self, I, J):
        return (I % self.P) * self.Q + (J % self.Q)

    @staticmethod
    def first_at_least(x, r, S):
        """Smallest local index i with i * S + r >= x."""
        return max(0, -(-(x - r) // S))

    def row_first(self, x, p=None):
        return self.first_at_least(x, self.p if p is None else p, self.P)

    def col_first(self, x, q=None):
        return self.first_at_least(x, self.q if q is None else q, self.Q)

    def piece_count(self, k, p):
        """Panel tiles I > k owned by process row p (piece p of iteration k)."""
        return max(0, len(range(p, self.nt, self.P)) - self.row_first(k + 1, p))

    def to_local(self, gi, gj):
        """Global element -> local element of its owner."""
        I, J = gi // self.nb, gj // self.nb
        return (I // self.P) * self.nb + gi % self.nb, (J // self.Q) * self.nb + gj % self.nb

    def lcol_sources(self, k):
        """For this rank's local trailing tile columns J > k (in order): the
        (piece, index in piece) of L_Jk."""
        out = []
        for jl in range(self.col_first(k + 1), self.nt_loc):
            J = jl * self.Q + self.q
            pp = J % self.P
            out.append((pp, J // self.P - self.row_first(k + 1, pp)))
        return out


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


def classify_bcast(nflag: int, nrecv: int) -> str:
    """L361-L363: of the nrecv receivers of one broadcast, nflag found (and
    corrected) corruption in their copy."""
    if nflag == 0:
        return "clean"
    return "restart" if nflag >= nrecv else "communication"


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
                  tmu_groups=32, restart=True):
    """Fault-tolerant lower Cholesky of the distributed matrix in place.
    A_loc: this rank's local column-major matrix (from scatter_tiles).
    inject: (iter, point, gi, gj, xor_mask, rank) with global (gi, gj);
    point in abft.AT_* (applied by the tile's owner) or AT_BCAST (applied to
    `rank`'s received copy of panel element (gi, gj) of iteration iter).
    Returns (rc, MgpuStats); rc is 0 or abft.E_UNCORRECTABLE."""
    nb, nt, P, Q = lay.nb, lay.nt, lay.P, lay.Q
    p, q = lay.p, lay.q
    dev, dt = A_loc.device, A_loc.dtype
    world = P * Q
    me = lay.rank
    tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, tol_scale, 1)
    mat = abft.Mat.alloc(A_loc, nb) if abft_on else abft.Mat(A_loc, nb)
    rep = abft.Report.alloc(mat) if abft_on else None
    rep_b = abft.Report(abft.colmajor_zeros(max(nt, 1), 1, dtype=torch.int32, device=dev),
                        torch.zeros(abft.NCOUNTS, dtype=torch.int32, device=dev))
    cb_total = torch.zeros(abft.NCOUNTS, dtype=torch.int32, device=dev)
    bflag = torch.zeros(nt, P + 1, dtype=torch.int32, device=dev)  # [k][piece | diag]
    consumed = torch.zeros(1, dtype=torch.int32, device=dev)
    fixes = torch.zeros(4096 * abft.FIX_BYTES, dtype=torch.uint8, device=dev)
    nfix = torch.zeros(1, dtype=torch.int32, device=dev)
    infos = torch.zeros(max(nt, 1), dtype=torch.int32, device=dev)
    Linv = abft.colmajor_zeros(nb, nb, dtype=dt, device=dev)
    diag_buf = _Piece(1, nb, dt, dev)

    def bcast(t, src):
        if world > 1:
            dist.broadcast(t, src=src, group=group)

    def check(m, tl, which):
        abft.abft_verify(m, tl, which, tol, rep)
        abft.abft_locate_correct(m, tl, which, tol, rep, fixes, nfix)

    def check_recv(m, tl, slot_k, slot):
        """Post-broadcast check of a received copy (L355); flags per source."""
        abft.abft_verify(m, tl, abft.COL, tol, rep_b)
        abft.abft_locate_correct(m, tl, abft.COL, tol, rep_b, fixes, nfix)
        bflag[slot_k, slot] += (rep_b.counts[0] > 0).to(torch.int32)
        cb_total.add_(rep_b.counts)
        rep_b.counts.zero_()

    def hook(k, point):
        for f in inject:
            it, pt, gi, gj, mask = f[:5]
            if it != k or pt != point or pt == AT_BCAST:
                continue
            if lay.owner(gi // nb, gj // nb) == me:
                li, lj = lay.to_local(gi, gj)
                abft.abft_inject(A_loc, li, lj, mask)

    def hook_bcast(k, buf: _Piece, tiles_I):
        """Communication fault: flip this rank's received copy."""
        for f in inject:
            it, pt, gi, gj, mask = f[:5]
            rk = f[5] if len(f) > 5 else -1
            if it != k or pt != AT_BCAST or rk != me or gj // nb != k or gi // nb not in tiles_I:
                continue
            t = tiles_I.index(gi // nb)
            abft.abft_inject(buf.L, t * nb + gi % nb, gj % nb, mask)

    restarts = [0]
    rs = abft_on and restart

    def snapshot(*ts):
        return [t.clone() for t in ts] + [rep.counts[abft.NCOUNTS - 1].clone()]

    def added_2d(snap):
        """2D errors the post-op check added (host read-back, f1)."""
        return int((rep.counts[abft.NCOUNTS - 1] - snap[-1]).item())

    def restore(snap, *ts):
        for t, c in zip(ts, snap[:-1]):
            t.copy_(c)
        rep.counts[abft.NCOUNTS - 1] = snap[-1]
        restarts[0] += 1

    def sub(m: abft.Mat, il, jl):
        """One local tile as its own 1x1-tile Mat (views into m's arrays)."""
        r0, c0 = il * nb, jl * nb
        return abft.Mat(m.A[r0:r0 + nb, c0:c0 + nb], nb,
                        m.colchk[2 * il:2 * il + 2, c0:c0 + nb] if m.colchk is not None else None,
                        m.rowchk[r0:r0 + nb, 2 * jl:2 * jl + 2] if m.rowchk is not None else None,
                        m.colmag[il:il + 1, c0:c0 + nb] if m.colmag is not None else None,
                        m.rowmag[r0:r0 + nb, jl:jl + 1] if m.rowmag is not None else None)

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
        # ---- 1. PD on the owner of A_kk
        if me == owner_kk:
            D = sub(mat, ik, jk)
            hook(k, abft.AT_PRE_PD_CHECK)
            if abft_on:
                check(D, abft.tiles(0, 1, 0, 1, False, abft.SYM_LOWER), abft.BOTH)
            if rs:
                pd_snap = snapshot(D.A, D.colchk, D.colmag)
            hook(k, abft.AT_PRE_PD)
            abft.abft_panel_potrf(D, infos[k:k + 1], Linv)
            hook(k, abft.AT_POST_PD)
            if abft_on:
                check(D, abft.tiles(0, 1, 0, 1, False, abft.LOWER), abft.COL)
            if rs and added_2d(pd_snap) > 0:  # local restart of the PD (L430)
                restore(pd_snap, D.A, D.colchk, D.colmag)
                abft.abft_panel_potrf(D, infos[k:k + 1], Linv)
                check(D, abft.tiles(0, 1, 0, 1, False, abft.LOWER), abft.COL)
            diag_buf.L.copy_(D.A)
            if abft_on:
                diag_buf.c.copy_(D.colchk)
                diag_buf.m.copy_(D.colmag)
        # ---- 2. broadcast L_kk to the panel's process column (sent to all)
        bcast(diag_buf.flat, owner_kk)
        if q == kq and me != owner_kk:
            hook_bcast(k, diag_buf, [k])
            if abft_on:
                check_recv(diag_buf.mat(), abft.tiles(0, 1, 0, 1, False, abft.LOWER), k, P)
            abft.abft_tri_inverse("L", "N", diag_buf.L, Linv)
        if k == nt - 1:
            break
        # ---- 3. PU on the panel owners
        ir0 = lay.row_first(k + 1)
        cnt = lay.mt_loc - ir0
        if q == kq and cnt > 0:
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
            pu()
            hook(k, abft.AT_POST_PU)
            if abft_on:
                check(mat, abft.tiles(ir0, lay.mt_loc, jk, jk + 1), abft.COL)
            if rs and added_2d(pu_snap) > 0:  # local restart of the PU (L430, L434)
                restore(pu_snap, *pan)
                pu()
                check(mat, abft.tiles(ir0, lay.mt_loc, jk, jk + 1), abft.COL)
        # ---- 4. broadcast the panel pieces (one per process row)
        pieces = []
        for pp in range(P):
            c_pp = lay.piece_count(k, pp)
            buf = _Piece(c_pp, nb, dt, dev) if c_pp else None
            pieces.append(buf)
            if not c_pp:
                continue
            src = pp * Q + kq
            if me == src:
                buf.L.copy_(A_loc[ir0 * nb:, jk * nb:(jk + 1) * nb])
                if abft_on:
                    buf.c.copy_(mat.colchk[2 * ir0:, jk * nb:(jk + 1) * nb])
                    buf.m.copy_(mat.colmag[ir0:, jk * nb:(jk + 1) * nb])
            bcast(buf.flat, src)
            if me != src:
                first = lay.row_first(k + 1, pp)
                tiles_I = [(first + t) * P + pp for t in range(c_pp)]
                hook_bcast(k, buf, tiles_I)
                if abft_on:
                    check_recv(buf.mat(), abft.tiles(0, c_pp, 0, 1), k, pp)
        # ---- 5. trailing update of the local tiles I >= J > k
        srcs = lay.lcol_sources(k)
        ncol = len(srcs)
        Lrow = pieces[p]
        if ncol and Lrow is not None:
            Lcol = _Piece(ncol, nb, dt, dev)
            for pp in range(P):
                sel = [t for t, (s, _) in enumerate(srcs) if s == pp]
                if not sel:
                    continue
                dst_idx = torch.tensor(sel, device=dev)
                src_idx = torch.tensor([srcs[t][1] for t in sel], device=dev)
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
                    abft.abft_verify(buf.mat(), abft.tiles(0, buf.cnt, 0, 1), abft.COL, tol, rep_b)
                    abft.abft_locate_correct(buf.mat(), abft.tiles(0, buf.cnt, 0, 1), abft.COL, tol, rep_b, fixes,
                                             nfix)
                consumed.add_(nfix - before)
                cb_total.add_(rep_b.counts)
                rep_b.counts.zero_()
        elif ncol == 0 or Lrow is None:
            hook(k, abft.AT_PRE_TMU)
            hook(k, abft.AT_POST_TMU)
        # ---- 6b. the panel owners' stored pieces (the factor itself): Alg. 2
        # line 13 re-checks the panel after the TMU; here the update read the
        # broadcast copies (checked above), so a fault in the stored piece
        # since its post-PU check was consumed by nobody and is a plain fix
        if abft_on and q == kq and cnt > 0:
            check(mat, abft.tiles(ir0, lay.mt_loc, jk, jk + 1), abft.COL)

    # ---- error reports: one all-reduce of the int32 counters (L361-L363)
    rep_counts = rep.counts if rep is not None else torch.zeros(abft.NCOUNTS, dtype=torch.int32, device=dev)
    nrs = torch.tensor([restarts[0]], dtype=torch.int32, device=dev)
    summary = torch.cat([rep_counts, cb_total, consumed, infos, bflag.reshape(-1), nrs])
    if world > 1:
        dist.all_reduce(summary, op=dist.ReduceOp.SUM, group=group)
    h = summary.cpu().tolist()
    st = MgpuStats()
    st.counts = h[:8]
    st.bcast_counts = h[8:16]
    st.tmu_consumed = h[16]
    inf = h[17:17 + nt]
    bf = h[17 + nt:-1]
    st.restarts = h[-1]
    for kk in range(nt):
        if inf[kk] and not st.info:
            st.info = kk * nb + inf[kk]
        for slot in range(P + 1):
            nflag = bf[kk * (P + 1) + slot]
            if nflag:
                nrecv = (P - 1) if slot == P else world - 1  # diag: the rest of process column k
                st.bcast_events.append((kk, slot, nflag, nrecv, classify_bcast(nflag, nrecv)))
    st.uncorrectable = st.counts[abft.NCOUNTS - 1] + st.bcast_counts[abft.NCOUNTS - 1] + st.tmu_consumed
    rc = abft.E_UNCORRECTABLE if st.uncorrectable else 0
    return rc, st
