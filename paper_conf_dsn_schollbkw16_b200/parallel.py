"""Row-block sharding of the protected SpMV across ranks (one process per GPU).

SURVEY.md §8(e): the rows of A are split into contiguous, 32-row-aligned
ranges; row blocks never straddle ranks, so C's rows, the detection and the
correction stay rank-local.  Each call needs one exchange step (the x halo)
and one scalar reduction (beta = ||x||_2):

* Local column numbering keeps GLOBAL order: the columns a rank references
  are sorted, so its x vector is laid out [halo below | own rows | halo above]
  and every pairwise sum (R2) sees the same operands in the same
  order as on one GPU -- y, t1, t2, s and the flags are bit-identical.
* The halo comes from the owning ranks over NCCL point-to-point (NVLink /
  NVSwitch on the B200 box; gloo in the CPU tests).  Owned ranges are
  contiguous, so each neighbour's halo is one contiguous slice of the local x.
* beta: each rank's PW sum of its own x_i^2 is an aligned node of the global
  PW tree when the ranges are equal powers of two; the partials are
  all-gathered (8 bytes per rank) and finished in rank order on the device
  (abft_finish) -- the single-GPU beta bit for bit.

The host logic here is plain data movement (partitioning, renumbering, index
lists); every step of the method itself runs in libabft.so.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import inputs as G


def block_partition(n: int, world: int, align: int = 32) -> list[tuple[int, int]]:
    """Contiguous row ranges, boundaries multiples of `align` (the last range
    takes the remainder).  Equal power-of-two ranges keep beta bit-exact."""
    groups = (n + align - 1) // align
    out, g0 = [], 0
    for r in range(world):
        g1 = groups * (r + 1) // world
        out.append((min(g0 * align, n), min(g1 * align, n)))
        g0 = g1
    return out


@dataclass
class Shard:
    """The local view of one rank: rows [row0, row1) of the global matrix."""
    rank: int
    world: int
    row0: int
    row1: int
    csr: G.CSR                # local rows, local (global-order) column indices
    n_cols: int               # local columns = len(cols)
    x_offset: int             # local index of global row0
    cols: np.ndarray          # global index of each local column (sorted)
    recv: dict = field(default_factory=dict)   # q -> (local start, count): halo from rank q
    send: dict = field(default_factory=dict)   # q -> local own indices rank q needs

    @property
    def n(self) -> int:
        return self.row1 - self.row0


def make_shard(rows: G.CSR, row0: int, row1: int, rank: int, world: int,
               ranges: list[tuple[int, int]]) -> Shard:
    """Renumber a rank's rows (global column indices) to the local layout
    [halo below | own | halo above] in global order and record, per owning
    rank, the contiguous local slice its halo lands in."""
    own = np.arange(row0, row1, dtype=np.int64)
    ref = np.unique(rows.col.astype(np.int64))
    cols = np.union1d(ref, own)
    local = np.searchsorted(cols, rows.col.astype(np.int64)).astype(np.int32)
    x_offset = int(np.searchsorted(cols, row0))
    sh = Shard(rank, world, row0, row1, G.CSR(rows.row_ptr, local, rows.val, rows.name),
               int(cols.shape[0]), x_offset, cols)
    for q, (a, b) in enumerate(ranges):
        if q == rank or a == b:
            continue
        lo, hi = np.searchsorted(cols, a), np.searchsorted(cols, b)
        if hi > lo:
            sh.recv[q] = (int(lo), int(hi - lo))
    return sh


def exchange_plans(shards_or_needs, ranks) -> None:
    """Given every rank's shard (or, distributed, the gathered halo needs),
    fill each shard's send lists: rank r sends to q the own entries q needs,
    in q's (global) order."""
    by_rank = {sh.rank: sh for sh in shards_or_needs}
    for q in ranks:
        shq = by_rank[q]
        for r, (start, count) in shq.recv.items():
            need = shq.cols[start:start + count]          # global indices owned by r
            shr = by_rank[r]
            shr.send[q] = (need - shr.row0 + shr.x_offset).astype(np.int64)


def plan_from_needs(sh: Shard, needs: dict) -> None:
    """Distributed variant: `needs[q]` = the global indices rank q needs from
    this rank (gathered from all ranks)."""
    for q, need in needs.items():
        sh.send[q] = (np.asarray(need, dtype=np.int64) - sh.row0 + sh.x_offset)


def halo_needs(sh: Shard) -> dict:
    """Global indices this rank needs from each owning rank."""
    return {q: sh.cols[s:s + c].tolist() for q, (s, c) in sh.recv.items()}


# ---------------------------------------------------------------------------
# Distributed protected SpMV on top of the C ABI (include/abft.h "Multi-GPU"):
# the library builds the shard's column order and halo plan, packs the send
# buffers with the x^2 partial, and -- with an NCCL communicator -- does the
# exchange itself (abft_dist_spmv, abft_dist_pcg).  Without a communicator
# (tests: logical ranks on one GPU, or processes over gloo) the exchange
# classes below move the library's buffers: abft_dist_begin -> copies ->
# abft_dist_end.
# ---------------------------------------------------------------------------
def shard_rows(A: G.CSR, a: int, b: int) -> G.CSR:
    """Rows [a, b) of A with their GLOBAL column indices."""
    return G.CSR(A.row_ptr[a:b + 1] - A.row_ptr[a], A.col[A.row_ptr[a]:A.row_ptr[b]],
                 A.val[A.row_ptr[a]:A.row_ptr[b]])


def ranges_array(ranges) -> np.ndarray:
    """[(a, b), ...] -> the [world + 1] boundary array abft_dist_create takes."""
    return np.array([ranges[0][0]] + [b for _, b in ranges], dtype=np.int64)


@dataclass
class ShardInfo:
    rank: int
    world: int
    row0: int
    row1: int

    @property
    def n(self) -> int:
        return self.row1 - self.row0


class DistSpmv:
    """One rank's shard: a DistHandle over its rows (global columns), the
    result y and the gathered partials (external exchange)."""

    def __init__(self, dist, rows: G.CSR, block_size: int = 32, max_rounds: int = 4,
                 device="cuda"):
        import torch

        from .abft import CsrDevice
        self.dist = dist
        self.sh = ShardInfo(dist.rank, dist.world, dist.row0, dist.row1)
        self.A = CsrDevice(rows.n, torch.from_numpy(np.ascontiguousarray(rows.row_ptr)).to(device),
                           torch.from_numpy(np.ascontiguousarray(rows.col)).to(device),
                           torch.from_numpy(np.ascontiguousarray(rows.val)).to(device))
        self.h = dist.encode(self.A, block_size, max_rounds)
        self.max_rounds = max_rounds
        self.y = torch.empty(rows.n, dtype=torch.float64, device=device)
        self.parts = torch.zeros(dist.world, dtype=torch.float64, device=device)

    def own_ptr(self) -> int:
        return self.h.own_ptr()

    def set_own(self, x_own) -> None:
        """Write this rank's x into the operand's own slice."""
        from .abft import lib
        lib().abft_memcpy(self.own_ptr(), x_own.data_ptr(), 8 * self.sh.n, None)

    def spmv(self, exchange=None, x_own=None, inject=None, mode=None):
        """One distributed protected SpMV (all ranks call it): over the
        library's NCCL communicator, or through `exchange` (external)."""
        from .abft import AUTOCORRECT, CHECK
        mode = CHECK | AUTOCORRECT if mode is None else mode
        if self.dist.nccl:
            return self.h.dist_spmv(x_own, self.y, inject, mode)
        return exchange.spmv(self, x_own, inject, mode)

    def plain(self, exchange=None, x_own=None):
        from .abft import NOCHECK
        return self.spmv(exchange, x_own, None, NOCHECK)


class LocalExchange:
    """Logical ranks in one process (tests on one GPU): the send lists come
    from the other shards' needs; every SpMV runs begin on all ranks, moves
    each send slice into its peer's receive slice and all partials into every
    rank's parts array (rank order), then end on all ranks."""

    def __init__(self, dss):
        self.dss = {d.sh.rank: d for d in dss}
        for r, d in self.dss.items():
            for q, dq in self.dss.items():
                if q != r:
                    d.h.set_send(q, dq.h.needs(r))

    def halo(self, x_owns=None):
        """begin on every rank (x_owns: rank -> tensor or None) + the copies."""
        import torch

        from .abft import lib
        for r, d in self.dss.items():
            d.h.begin(None if x_owns is None else x_owns.get(r))
        torch.cuda.synchronize()
        for r, d in self.dss.items():
            for q, dq in self.dss.items():
                if q == r:
                    continue
                sp, sc, _, _ = d.h.buffers(q)
                _, _, rp, rc = dq.h.buffers(r)
                assert sc == rc, (r, q, sc, rc)
                if sc:
                    lib().abft_memcpy(rp, sp, 8 * sc, None)
        for r, d in self.dss.items():
            for q, dq in self.dss.items():
                lib().abft_memcpy(dq.parts.data_ptr() + 8 * r, d.h.partial_ptr(), 8, None)

    def spmv(self, ds, x_own, inject, mode):
        raise RuntimeError("logical ranks step together: use spmv_all")

    def spmv_all(self, x_owns=None, injects=None, mode=None):
        from .abft import AUTOCORRECT, CHECK
        mode = CHECK | AUTOCORRECT if mode is None else mode
        self.halo(x_owns)
        for r, d in self.dss.items():
            d.h.end(d.y, d.parts, None if injects is None else injects.get(r), mode)
        return {r: d.y for r, d in self.dss.items()}


class TorchExchange:
    """One process per rank over torch.distributed without the library's
    communicator (tests: gloo, several processes sharing one GPU): the needs
    are all-gathered once, each SpMV stages the library's send / receive
    slices through host tensors."""

    def __init__(self, ds: DistSpmv, group=None):
        import torch.distributed as dist
        self.dist, self.group = dist, group
        self.rank, self.world = dist.get_rank(group), dist.get_world_size(group)
        mine = {q: ds.h.needs(q).tolist() for q in range(self.world) if q != self.rank}
        allneeds = [None] * self.world
        dist.all_gather_object(allneeds, mine, group=group)
        for q in range(self.world):
            if q != self.rank:
                ds.h.set_send(q, allneeds[q].get(self.rank, []))

    def _d2h(self, ptr, count):
        import torch

        from .abft import lib
        t = torch.empty(count, dtype=torch.float64)
        if count:
            lib().abft_memcpy(t.data_ptr(), ptr, 8 * count, None)
        return t

    def _h2d(self, ptr, t):
        from .abft import lib
        if t.numel():
            lib().abft_memcpy(ptr, t.data_ptr(), 8 * t.numel(), None)

    def gather(self, send_dev, recv_dev) -> None:
        """All-gather a device vector (rank order) through the host."""
        import torch
        s = send_dev.cpu()
        out = torch.empty(s.numel() * self.world, dtype=torch.float64)
        self.dist.all_gather_into_tensor(out, s, group=self.group)
        recv_dev.copy_(out.to(recv_dev.device))

    def spmv(self, ds, x_own, inject, mode):
        import torch
        h = ds.h
        h.begin(x_own)
        torch.cuda.synchronize()
        ops, recvs = [], []
        for q in range(self.world):
            if q == self.rank:
                continue
            sp, sc, rp, rc = h.buffers(q)
            if sc:
                ops.append(self.dist.P2POp(self.dist.isend, self._d2h(sp, sc), q, self.group))
            if rc:
                t = torch.empty(rc, dtype=torch.float64)
                recvs.append((rp, t))
                ops.append(self.dist.P2POp(self.dist.irecv, t, q, self.group))
        if ops:
            for w in self.dist.batch_isend_irecv(ops):
                w.wait()
        for rp, t in recvs:
            self._h2d(rp, t)
        part = self._d2h(h.partial_ptr(), 1)
        out = torch.empty(self.world, dtype=torch.float64)
        self.dist.all_gather_into_tensor(out, part, group=self.group)
        ds.parts.copy_(out.to(ds.parts.device))
        h.end(ds.y, ds.parts, inject, mode)
        return ds.y


# ---------------------------------------------------------------------------
# Distributed Jacobi-PCG on top of the C ABI
# ---------------------------------------------------------------------------
class DistPcg:
    """One rank's share of the distributed PCG.  With the library's NCCL
    communicator the whole solve is abft_dist_pcg (every exchange inside the
    library).  Without one (tests) this class sequences the same device
    phases (abft_pcg_dist_*) around an external exchange: the x halo of every
    SpMV and the all-gather of the per-phase dot partials (3 doubles per
    rank), finished in rank order on the device (R28)."""

    def __init__(self, ds: DistSpmv, check: bool = True, variant: str = "pcg", inject=None):
        import torch
        if variant not in ("pcg", "cg1"):
            raise ValueError(variant)
        if inject is not None and not check:
            raise ValueError("fault injection needs the protected SpMV")
        self.ds, self.check, self.variant, self.inject = ds, check, variant, inject
        self.calls = 0
        dev = ds.y.device
        world = ds.sh.world
        self.send = torch.zeros(3, dtype=torch.float64, device=dev)
        self.recv = torch.zeros(3 * world, dtype=torch.float64, device=dev)

    def begin(self, b, x, n_global, tol=1e-6, max_iter=0, res_hist=None, diag=None):
        mi = max_iter if max_iter > 0 else 10 * n_global
        self.x, self.mi, self.calls = x, mi, 0
        self.ds.h.pcg_dist_begin(b, x, self.ds.own_ptr(), self.ds.y, diag, tol, mi, self.check,
                                 res_hist)
        self.ds.set_own(x)  # the first SpMV operand is x0
        return mi

    def next_inject(self):
        inj = self.inject(self.calls) if self.inject is not None else None
        self.calls += 1
        return inj

    def mode(self):
        from .abft import AUTOCORRECT, CHECK, NOCHECK
        return CHECK | AUTOCORRECT if self.check else NOCHECK

    def local(self, phase, it=0):
        from .abft import PCG_PHASE_P
        self.ds.h.pcg_dist_local(phase, it, None if phase == PCG_PHASE_P else self.send)
        return self.send

    def combine(self, phase, it=0):
        self.ds.h.pcg_dist_combine(phase, it, self.recv, self.ds.sh.world)

    def status(self):
        return self.ds.h.pcg_dist_status()

    def run(self, spmv, reduce, local, status, mi, poll=16):
        """Sequence one solve (after begin).  spmv(): the distributed SpMV of
        the operand's own slice into ds.y; reduce(phases): run each
        (phase, it) local kernel, gather the send slots, combine the last
        phase; local(phase, it): a kernel without a reduction; status():
        (state, stats).  variant "pcg": standard (two reductions per
        iteration); "cg1": single reduction (Chronopoulos-Gear, R29)."""
        from .abft import (PCG_PHASE_CG1_DOT, PCG_PHASE_CG1_UPDATE, PCG_PHASE_DOT,
                           PCG_PHASE_INIT, PCG_PHASE_P, PCG_PHASE_UPDATE)
        spmv()
        reduce([(PCG_PHASE_INIT, 0)])
        if self.variant == "cg1":
            spmv()  # w_0 = A u_0
            reduce([(PCG_PHASE_CG1_DOT, 0)])
        j = 0
        while True:
            state = status()
            if state[0] != 0 or j >= mi:
                return state
            for it in range(j + 1, j + min(poll, mi - j) + 1):
                if self.variant == "cg1":
                    local(PCG_PHASE_CG1_UPDATE, it)
                    spmv()  # w = A u
                    reduce([(PCG_PHASE_CG1_DOT, it)])
                else:
                    spmv()  # q = A p (p sits in the operand's own slice)
                    reduce([(PCG_PHASE_DOT, it)])
                    reduce([(PCG_PHASE_UPDATE, it)])
                    local(PCG_PHASE_P, it)
            j += min(poll, mi - j)

    def solve(self, exchange, b, x, n_global, tol=1e-6, max_iter=0, res_hist=None, diag=None,
              poll=16):
        """One solve: abft_dist_pcg over the library's communicator, or the
        phases over `exchange` (a TorchExchange)."""
        if self.ds.dist.nccl:
            inj = self.inject(0) if self.inject is not None else None
            status, st = self.ds.h.dist_pcg(b, x, diag, tol, max_iter, inj, self.check, res_hist,
                                            variant=self.variant)
            return {0: 1, -5: 3, -7: 2}.get(status, status), st

        def spmv():
            exchange.spmv(self.ds, None, self.next_inject(), self.mode())

        def reduce(phases):
            for ph, it in phases:
                self.local(ph, it)
            exchange.gather(self.send, self.recv)
            self.combine(*phases[-1])

        mi = self.begin(b, x, n_global, tol, max_iter, res_hist, diag)
        return self.run(spmv, reduce, self.local, self.status, mi, poll)


def pcg_lockstep(pcgs, exchange: LocalExchange, bs, xs, n_global, tol=1e-6, max_iter=0,
                 hists=None, poll=16):
    """Logical ranks in one process (tests): every phase runs on all ranks,
    then the partials are concatenated in rank order -- the exchange pattern
    of DistPcg.solve without a process group.  Rank 0's DistPcg.run sequences
    the solve; its callbacks act on every rank."""
    import torch
    hists = hists or [None] * len(pcgs)

    def spmv():
        injects = {p.ds.sh.rank: p.next_inject() for p in pcgs}
        exchange.spmv_all(None, injects, pcgs[0].mode())

    def reduce(phases):
        for p in pcgs:
            for ph, it in phases:
                p.local(ph, it)
        sends = torch.cat([p.send for p in pcgs])
        for p in pcgs:
            p.recv.copy_(sends)
            p.combine(*phases[-1])

    def local(phase, it=0):
        for p in pcgs:
            p.local(phase, it)

    mi = 0
    for p, b, x, h in zip(pcgs, bs, xs, hists):
        mi = p.begin(b, x, n_global, tol, max_iter, h)
    pcgs[0].run(spmv, reduce, local, pcgs[0].status, mi, poll)
    return [p.status() for p in pcgs]
