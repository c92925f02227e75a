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
# Exchange backends (x_ext: the local extended vector, a torch tensor)
# ---------------------------------------------------------------------------
class TorchDistComm:
    """Halo exchange with torch.distributed point-to-point (NCCL on GPUs,
    gloo on CPU) and the beta partials with all_gather_into_tensor."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self._idx = {}
        # gloo carries CPU tensors only: stage device buffers through the host
        self.stage = dist.get_backend(group) != "nccl"

    def halo(self, sh: Shard, x_ext) -> None:
        import torch
        stage = self.stage and x_ext.is_cuda
        ops, bufs, recvs = [], [], []
        for q, idx in sorted(sh.send.items()):
            key = (id(sh), q, x_ext.device)
            if key not in self._idx:
                self._idx[key] = torch.as_tensor(idx, device=x_ext.device)
            buf = x_ext.index_select(0, self._idx[key])
            if stage:
                buf = buf.cpu()
            bufs.append(buf)
            ops.append(self.dist.P2POp(self.dist.isend, buf, q, self.group))
        for q, (start, count) in sorted(sh.recv.items()):
            dst = x_ext[start:start + count]
            if stage:
                tmp = torch.empty(count, dtype=x_ext.dtype)
                recvs.append((dst, tmp))
                dst = tmp
            ops.append(self.dist.P2POp(self.dist.irecv, dst, q, self.group))
        if ops:
            for w in self.dist.batch_isend_irecv(ops):
                w.wait()
        for dst, tmp in recvs:
            dst.copy_(tmp)

    def gather_partials(self, partial, out) -> None:
        if self.stage and partial.is_cuda:
            o = out.cpu()
            self.dist.all_gather_into_tensor(o, partial.cpu(), group=self.group)
            out.copy_(o)
        else:
            self.dist.all_gather_into_tensor(out, partial, group=self.group)

    def gather_needs(self, sh: Shard) -> dict:
        """All-to-all of halo needs (once, at setup)."""
        mine = halo_needs(sh)
        allneeds = [None] * self.world
        self.dist.all_gather_object(allneeds, mine, group=self.group)
        return {q: allneeds[q][sh.rank] for q in range(self.world)
                if q != sh.rank and sh.rank in allneeds[q]}


class LocalComm:
    """All shards in one process (logical shards on one GPU, tests): the halo
    is copied from the owners' extended vectors."""

    def __init__(self, shards, xs):
        self.shards = {s.rank: s for s in shards}
        self.xs = xs  # rank -> x_ext tensor
        self._idx = {}  # device index lists, uploaded once (graph capture safe)

    def halo(self, sh: Shard, x_ext) -> None:
        import torch
        for q, (start, count) in sh.recv.items():
            src = self.xs[q]
            key = (q, sh.rank, src.device)
            if key not in self._idx:
                self._idx[key] = torch.as_tensor(self.shards[q].send[sh.rank], device=src.device)
            x_ext[start:start + count] = src.index_select(0, self._idx[key])


# ---------------------------------------------------------------------------
# Distributed protected SpMV on top of the C ABI
# ---------------------------------------------------------------------------
class DistSpmv:
    """One rank's protected SpMV: halo exchange, fused multiply+detect on the
    local shard (ABFT_DEFER_FINISH), beta partial, all-gather, finish."""

    def __init__(self, shard: Shard, block_size: int = 32, max_rounds: int = 4,
                 device="cuda"):
        import torch

        from .abft import CsrDevice, Handle
        self.sh = shard
        A = CsrDevice(shard.n, torch.from_numpy(shard.csr.row_ptr).to(device),
                      torch.from_numpy(shard.csr.col).to(device),
                      torch.from_numpy(shard.csr.val).to(device),
                      n_cols=shard.n_cols, x_offset=shard.x_offset)
        self.h = Handle(A, block_size, max_rounds)
        self.max_rounds = max_rounds
        self.x_ext = torch.zeros(shard.n_cols, dtype=torch.float64, device=device)
        self.y = torch.empty(shard.n, dtype=torch.float64, device=device)
        self.parts = torch.empty(shard.world, dtype=torch.float64, device=device)

    def own(self):
        s = self.sh
        return self.x_ext[s.x_offset:s.x_offset + s.n]

    def step1(self, comm, inject=None):
        """Halo + fused pass (steps 1-3) + this rank's beta partial."""
        import torch

        from .abft import CHECK, DEFER_FINISH
        comm.halo(self.sh, self.x_ext)
        self.h.spmv(self.x_ext, self.y, inject=inject, mode=CHECK | DEFER_FINISH)
        if not hasattr(self, "_part"):
            self._part = torch.empty(1, dtype=torch.float64, device=self.x_ext.device)
        return self.h.beta_partial(self._part)

    def spmv(self, comm, inject=None, rounds=None):
        """One distributed protected SpMV (all ranks call it)."""
        part = self.step1(comm, inject)
        comm.gather_partials(part, self.parts)
        return self.step2(rounds, inject)

    def step2(self, rounds=None, inject=None):
        """Steps 4-5 with beta from all ranks' partials (self.parts)."""
        self.h.finish(self.x_ext, self.y, self.parts, rounds, inject)
        return self.y

    def plain(self, comm):
        """Unprotected SpMV (same kernels, check off) over the extended x."""
        from .abft import NOCHECK
        comm.halo(self.sh, self.x_ext)
        self.h.spmv(self.x_ext, self.y, mode=NOCHECK)
        return self.y


# ---------------------------------------------------------------------------
# Distributed Jacobi-PCG on top of the C ABI
# ---------------------------------------------------------------------------
class DistPcg:
    """One rank's share of the distributed PCG.  Vector kernels and scalar
    updates run in libabft.so (abft_pcg_dist_*); this class only sequences
    them around the two exchanges: the x halo of every SpMV (DistSpmv) and the
    all-gather of the per-phase dot partials (3 doubles per rank), finished in
    rank order on the device (R28).  Iterates like abft_pcg: the
    device state word is read every `poll` iterations; every rank computes
    identical scalars from identical partials, so all stop together."""

    def __init__(self, ds: DistSpmv, check: bool = True, variant: str = "pcg", inject=None):
        import torch
        if variant not in ("pcg", "cg1"):
            raise ValueError(variant)
        if inject is not None and not check:
            raise ValueError("fault injection needs the protected SpMV")
        self.ds, self.check, self.variant, self.inject = ds, check, variant, inject
        self.calls, self._inj = 0, None
        dev = ds.x_ext.device
        world = ds.sh.world
        self.send = torch.zeros(3, dtype=torch.float64, device=dev)
        self.recv = torch.zeros(3 * world, dtype=torch.float64, device=dev)

    def begin(self, b, x, n_global, tol=1e-6, max_iter=0, res_hist=None, diag=None):
        mi = max_iter if max_iter > 0 else 10 * n_global
        self.x, self.mi, self.calls = x, mi, 0
        self.ds.h.pcg_dist_begin(b, x, self.ds.own(), self.ds.y, diag, tol, mi, self.check,
                                 res_hist)
        self.ds.own().copy_(x)  # the first SpMV operand is x0
        return mi

    # -- the phases, each rank's half of one exchange --------------------------
    def spmv_local(self, comm):
        """Steps 1-3 of the SpMV (halo + fused pass); returns the beta partial
        to gather (None for the unprotected baseline).  With `inject` set
        (a function of the solve's SpMV call index -> Inject or None), the
        call's faults go into the protected pass and its correction rounds."""
        self._inj = self.inject(self.calls) if self.inject is not None else None
        self.calls += 1
        if not self.check:
            self.ds.plain(comm)
            return None
        return self.ds.step1(comm, self._inj)

    def spmv_finish(self):
        if self.check:
            self.ds.step2(None, self._inj)

    def local(self, phase, it=0):
        from .abft import PCG_PHASE_P
        self.ds.h.pcg_dist_local(phase, it, None if phase == PCG_PHASE_P else self.send)
        return self.send

    def combine(self, phase, it=0):
        self.ds.h.pcg_dist_combine(phase, it, self.recv, self.ds.sh.world)

    def status(self):
        return self.ds.h.pcg_dist_status()

    # -- the iteration, over any exchange ------------------------------------
    def run(self, spmv, reduce, local, status, mi, poll=16, graph=False, graph_key=None):
        """Sequence one solve (after begin).  spmv(): the distributed SpMV of
        the operand's own slice into ds.y; reduce(phases): run each
        (phase, it) local kernel, gather the send slots, combine the last
        phase; local(phase, it): a kernel without a reduction; status():
        (state, stats).  variant "pcg": standard (two reductions per
        iteration); "cg1": single reduction (Chronopoulos-Gear, R29).
        graph: capture `poll` iterations once and replay them (fault-free
        solves; every call in an iteration must be capturable)."""
        from .abft import (PCG_PHASE_CG1_DOT, PCG_PHASE_CG1_UPDATE, PCG_PHASE_DOT,
                           PCG_PHASE_INIT, PCG_PHASE_P, PCG_PHASE_UPDATE)
        spmv()
        reduce([(PCG_PHASE_INIT, 0)])
        if self.variant == "cg1":
            spmv()  # w_0 = A u_0
            reduce([(PCG_PHASE_CG1_DOT, 0)])
        def batch(j0, count):
            for j in range(j0 + 1, j0 + count + 1):
                if self.variant == "cg1":
                    local(PCG_PHASE_CG1_UPDATE, j)
                    spmv()  # w = A u
                    reduce([(PCG_PHASE_CG1_DOT, j)])
                else:
                    spmv()  # q = A p (p sits in the operand's own slice)
                    reduce([(PCG_PHASE_DOT, j)])
                    reduce([(PCG_PHASE_UPDATE, j)])
                    local(PCG_PHASE_P, j)

        j, g = 0, None
        if graph and graph_key is not None and getattr(self, "_graph", (None,))[0] == graph_key:
            g = self._graph[1]  # same buffers and launch arguments: replay the cached graph
        while True:
            state = status()
            if state[0] != 0 or j >= mi:
                return state
            if graph and mi - j >= poll:
                # One CUDA graph of `poll` iterations, replayed until the
                # device state leaves RUN.  The baked iteration indices
                # 1..poll only pair each update with its p step (upd ==
                # iter); kernels of a finished solve are no-ops and the host
                # never replays after one, so reuse is exact.
                if g is None:
                    # capture_begin/end directly: torch.cuda.graph() would
                    # also run gc.collect() + empty_cache() on every solve
                    import torch
                    g = torch.cuda.CUDAGraph()
                    cs = torch.cuda.Stream()
                    cs.wait_stream(torch.cuda.current_stream())
                    with torch.cuda.stream(cs):
                        g.capture_begin()
                        try:
                            batch(0, poll)
                        finally:
                            g.capture_end()
                    torch.cuda.current_stream().wait_stream(cs)
                    if graph_key is not None:
                        self._graph = (graph_key, g)
                g.replay()
                j += poll
            else:
                n = min(poll, mi - j)
                batch(j, n)
                j += n

    # -- driver over torch.distributed (one process per GPU) -----------------
    def solve(self, comm: TorchDistComm, b, x, n_global, tol=1e-6, max_iter=0, res_hist=None,
              diag=None, poll=16, graph=False):
        def spmv():
            part = self.spmv_local(comm)
            if part is not None:
                comm.gather_partials(part, self.ds.parts)
                self.spmv_finish()

        def reduce(phases):
            for ph, it in phases:
                self.local(ph, it)
            comm.gather_partials(self.send, self.recv)
            self.combine(*phases[-1])

        if graph and self.inject is not None:
            raise ValueError("graph replay needs a fault-free solve (per-call fault plans)")
        mi = self.begin(b, x, n_global, tol, max_iter, res_hist, diag)
        # the captured launches bake every pointer and the handle's argument
        # block: a later solve on the same buffers may replay the same graph
        key = (tuple(None if t is None else t.data_ptr() for t in (b, x, res_hist, diag)) +
               (tol, mi, poll)) if graph else None
        return self.run(spmv, reduce, self.local, self.status, mi, poll, graph, key)


def pcg_lockstep(pcgs, comm: LocalComm, bs, xs, n_global, tol=1e-6, max_iter=0, hists=None,
                 poll=16, graph=False):
    """Logical ranks in one process (tests): every phase runs on all ranks,
    then the partials are concatenated in rank order -- the exchange pattern
    of DistPcg.solve without a process group.  Rank 0's DistPcg.run sequences
    the solve; its callbacks act on every rank."""
    import torch
    hists = hists or [None] * len(pcgs)

    def spmv():
        parts = [p.spmv_local(comm) for p in pcgs]
        if parts[0] is not None:
            allp = torch.cat(parts)
            for p in pcgs:
                p.ds.parts.copy_(allp)
                p.spmv_finish()

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
    pcgs[0].run(spmv, reduce, local, pcgs[0].status, mi, poll, graph)
    return [p.status() for p in pcgs]
