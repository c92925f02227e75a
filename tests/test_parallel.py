"""Row-block sharding -- host logic on CPU.

* in-process: every shard's local (global-order) CSR, its halo and the
  oracle's SpMV / encoding on it reproduce the global oracle bit for bit;
  the PW of the per-rank x^2 partials equals the global one;
* 2 processes over gloo: the halo exchange and the partial all-gather.
"""
import os
import types

import numpy as np
import pytest

from paper_conf_dsn_schollbkw16_b200 import inputs as G
from paper_conf_dsn_schollbkw16_b200 import parallel as PL


def shard_all(A, world):
    ranges = PL.block_partition(A.n, world)
    shards = []
    for r, (a, b) in enumerate(ranges):
        rows = G.CSR(A.row_ptr[a:b + 1] - A.row_ptr[a], A.col[A.row_ptr[a]:A.row_ptr[b]],
                     A.val[A.row_ptr[a]:A.row_ptr[b]])
        shards.append(PL.make_shard(rows, a, b, r, world, ranges))
    PL.exchange_plans(shards, range(world))
    return ranges, shards


def halo_numpy(shards, x):
    """x_ext per shard assembled from the owners' send lists (as the comms do)."""
    ext = {}
    for sh in shards:
        e = np.zeros(sh.n_cols)
        e[sh.x_offset:sh.x_offset + sh.n] = x[sh.row0:sh.row1]
        ext[sh.rank] = e
    for sh in shards:
        for q, (start, count) in sh.recv.items():
            owner = shards[q]
            ext[sh.rank][start:start + count] = ext[q][owner.send[sh.rank]]
    return ext


def square(sh):
    """The shard as a square CSR (empty rows appended) for the oracle."""
    rp = np.concatenate([sh.csr.row_ptr, np.full(sh.n_cols - sh.n, sh.csr.row_ptr[-1])])
    return G.CSR(rp, sh.csr.col, sh.csr.val)


MATS = {"lap3d": lambda: G.laplacian_3d_7pt(8), "st27": lambda: G.stencil_3d_27pt(6, 6, 8),
        "rand": lambda: G.random_csr(256, 0.03, 5), "rmat": lambda: G.rmat(9, 8, 2)}


def test_partition_aligned():
    for n, w in [(4096, 2), (4096, 8), (1000, 3), (33, 4)]:
        r = PL.block_partition(n, w)
        assert r[0][0] == 0 and r[-1][1] == n
        for (a, b), (c, d) in zip(r, r[1:]):
            assert b == c and a % 32 == 0
    assert PL.block_partition(2 ** 21 * 4, 4) == [(i * 2 ** 21, (i + 1) * 2 ** 21) for i in range(4)]


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("name", sorted(MATS))
def test_shards_reproduce_global(O, name, world):
    A = MATS[name]()
    x = G.uniform_vector(A.n, 42)
    y = O.spmv(A, x)
    enc = O.encode(A, 32)
    ranges, shards = shard_all(A, world)
    ext = halo_numpy(shards, x)
    for sh in shards:
        # global order of local columns
        assert np.all(np.diff(sh.cols) > 0)
        assert np.array_equal(sh.cols[sh.csr.col], A.col[A.row_ptr[sh.row0]:A.row_ptr[sh.row1]])
        assert np.array_equal(ext[sh.rank], x[sh.cols])
        Ls = square(sh)
        yl = O.spmv(Ls, ext[sh.rank])[:sh.n]
        assert np.array_equal(yl.view(np.uint64), y[sh.row0:sh.row1].view(np.uint64))
        el = O.encode(Ls, 32)
        k0, nbl = sh.row0 // 32, (sh.n + 31) // 32
        for k in range(nbl):
            a, b = el.row_ptr[k], el.row_ptr[k + 1]
            ga, gb = enc.row_ptr[k0 + k], enc.row_ptr[k0 + k + 1]
            assert np.array_equal(sh.cols[el.col[a:b]], enc.col[ga:gb])
            assert np.array_equal(el.val[a:b].view(np.uint64), enc.val[ga:gb].view(np.uint64))
        assert np.array_equal(el.K[:nbl].view(np.uint64), enc.K[k0:k0 + nbl].view(np.uint64))
    # beta: PW of the per-rank partials == global PW (equal power-of-two ranges)
    if all((b - a) == ranges[0][1] - ranges[0][0] for a, b in ranges) and \
            (ranges[0][1] & (ranges[0][1] - 1)) == 0:
        parts = [O.pw(x[a:b] * x[a:b]) for a, b in ranges]
        assert O.pw(np.array(parts)) == O.pw(x * x)


@pytest.mark.parametrize("world", [1, 2, 3, 4])
@pytest.mark.parametrize("name", sorted(MATS))
def test_library_halo_plan_matches_reference(name, world):
    # abft_halo_plan (the host plan inside abft_dist_encode, C++) against the
    # independent numpy reference make_shard: local columns, halo slices
    from paper_conf_dsn_schollbkw16_b200 import halo_plan
    A = MATS[name]()
    ranges, shards = shard_all(A, world)
    rg = PL.ranges_array(ranges)
    for sh in shards:
        rows = PL.shard_rows(A, sh.row0, sh.row1)
        local, nb, na, rs, rc, halo = halo_plan(sh.rank, world, rg, rows.col)
        assert np.array_equal(local, sh.csr.col)
        assert nb == sh.x_offset and nb + sh.n + na == sh.n_cols
        assert np.array_equal(halo, np.concatenate([sh.cols[:nb], sh.cols[nb + sh.n:]]))
        for q in range(world):
            start, count = sh.recv.get(q, (0, 0))
            assert rc[q] == count and (count == 0 or rs[q] == start)


def _gloo_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist

    from paper_conf_dsn_schollbkw16_b200 import halo_plan
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = G.laplacian_3d_7pt(8)
        x = G.uniform_vector(A.n, 42)
        ranges = PL.block_partition(A.n, world)
        a, b = ranges[rank]
        rows = PL.shard_rows(A, a, b)
        # the library's host plan; needs exchanged over gloo (the protocol of
        # abft_dist_needs / abft_dist_set_send), then the halo itself
        local, nb, na, rs, rc, halo = halo_plan(rank, world, PL.ranges_array(ranges), rows.col)
        hb = np.concatenate([halo[:nb], np.zeros(b - a, np.int64), halo[nb:]])
        mine = {p: hb[rs[p]:rs[p] + rc[p]].tolist() for p in range(world) if p != rank and rc[p]}
        allneeds = [None] * world
        dist.all_gather_object(allneeds, mine)
        ext = torch.zeros(nb + (b - a) + na, dtype=torch.float64)
        ext[nb:nb + (b - a)] = torch.from_numpy(x[a:b])
        ops, bufs = [], []
        for p in range(world):
            if p == rank:
                continue
            need = allneeds[p].get(rank, [])
            if need:
                buf = torch.from_numpy(x[np.asarray(need)] * 1.0)
                assert np.all((np.asarray(need) >= a) & (np.asarray(need) < b))
                bufs.append(buf)
                ops.append(dist.P2POp(dist.isend, buf, p))
            if rc[p]:
                ops.append(dist.P2POp(dist.irecv, ext[rs[p]:rs[p] + rc[p]], p))
        if ops:
            for w in dist.batch_isend_irecv(ops):
                w.wait()
        cols = np.concatenate([halo[:nb], np.arange(a, b), halo[nb:]])
        ok = bool(np.array_equal(ext.numpy(), x[cols]))
        # the exchanged operand reproduces the global rows' products
        y = np.array([np.sum(rows.val[rows.row_ptr[i]:rows.row_ptr[i + 1]] *
                             ext.numpy()[local[rows.row_ptr[i]:rows.row_ptr[i + 1]]])
                      for i in range(b - a)])
        yg = np.array([np.sum(A.val[A.row_ptr[i]:A.row_ptr[i + 1]] *
                              x[A.col[A.row_ptr[i]:A.row_ptr[i + 1]]]) for i in range(a, b)])
        ok = ok and bool(np.array_equal(y, yg))
        part = torch.tensor([float(rank + 1)], dtype=torch.float64)
        out = torch.empty(world, dtype=torch.float64)
        dist.all_gather_into_tensor(out, part)
        ok = ok and out.tolist() == [float(r + 1) for r in range(world)]
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


def test_gloo_halo_exchange():
    import socket

    import torch.multiprocessing as mp
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: True, 1: True}


# ---------------------------------------------------------------------------
# Distributed PCG host protocol (parallel.DistPcg) on CPU: the device phases
# are replaced by a numpy test double with the semantics include/abft.h
# documents for abft_pcg_dist_*, so the sequencing, the halo of p / u and the
# rank-ordered partial gathers are exercised over real gloo processes and
# compared with the rank-partitioned oracle.
# ---------------------------------------------------------------------------
class _FakeHandle:
    def __init__(self, O):
        self.O = O

    def pcg_dist_begin(self, b, x, pext, q, diag, tol, mi, check, hist):
        self.b, self.x, self.pext, self.q = b.numpy(), x.numpy(), pext.numpy(), q.numpy()
        self.d = self.diag
        n = self.b.shape[0]
        self.r, self.z, self.p, self.s = (np.zeros(n) for _ in range(4))
        self.tol, self.mi, self.hist = tol, mi, hist
        self.sc = dict(state=0, it=0, rho=0.0, alpha=0.0, beta=0.0, calls=0, upd=-1)

    def pcg_dist_local(self, phase, it, send):
        O, sc = self.O, self.sc
        if phase not in (0, 3) and sc["state"] != 0:
            return
        sd = None if send is None else send.numpy()
        if phase == 0:
            self.r = self.b - self.q
            self.z = self.r / self.d
            self.p = self.z.copy()
            self.pext[:] = self.z
            sd[:3] = [O.pw(self.r * self.z), O.pw(self.r * self.r), O.pw(self.b * self.b)]
        elif phase == 1:
            sd[0] = O.pw(self.p * self.q)
        elif phase == 2:
            self.x[:] = self.x + sc["alpha"] * self.p
            self.r = self.r - sc["alpha"] * self.q
            self.z = self.r / self.d
            sd[:2] = [O.pw(self.r * self.z), O.pw(self.r * self.r)]
        elif phase == 3:
            if sc["upd"] == it:
                self.p = self.z + sc["beta"] * self.p
                self.pext[:] = self.p
        elif phase == 4:
            self.p = self.z + sc["beta"] * self.p
            self.s = self.q + sc["beta"] * self.s
            self.x[:] = self.x + sc["alpha"] * self.p
            self.r = self.r - sc["alpha"] * self.s
            self.z = self.r / self.d
            self.pext[:] = self.z
            sd[:2] = [O.pw(self.r * self.z), O.pw(self.r * self.r)]
        elif phase == 5:
            if it == 0:
                self.s = self.q.copy()
            sd[2] = O.pw(self.q * self.z)

    def pcg_dist_combine(self, phase, it, recv, world):
        O, sc = self.O, self.sc
        if phase != 0 and sc["state"] != 0:
            return
        rv = recv.numpy().reshape(world, 3)
        t = [O.pw(rv[:, c].copy()) for c in range(3)]
        sc["calls"] += 1 if phase in (0, 1, 5) else 0
        if phase == 0:
            sc["rho"], sc["res"] = t[0], np.sqrt(t[1])
            sc["thr"] = self.tol * np.sqrt(t[2])
            self.hist.append(sc["res"])
            sc["state"] = 1 if sc["res"] <= sc["thr"] else 0
        elif phase == 1:
            sc["alpha"] = sc["rho"] / t[0]
        elif phase == 2 or (phase == 5 and it > 0):
            ru, rr = t[0], t[1]
            sc["it"] += 1
            sc["res"] = np.sqrt(rr)
            self.hist.append(sc["res"])
            sc["upd"] = it
            if sc["res"] <= sc["thr"]:
                sc["state"] = 1
            elif sc["it"] >= self.mi:
                sc["state"] = 3
            elif phase == 2:
                sc["beta"], sc["rho"] = ru / sc["rho"], ru
            else:
                beta = ru / sc["rho"]
                den = t[2] - beta * ru / sc["alpha"]
                sc["beta"], sc["alpha"], sc["rho"] = beta, ru / den, ru
        else:  # cg1, iteration 0
            sc["alpha"], sc["beta"] = sc["rho"] / t[2], 0.0

    def pcg_dist_status(self):
        return self.sc["state"], {"iters": self.sc["it"], "spmv_calls": self.sc["calls"]}


class _FakeDs:
    """DistSpmv stand-in for DistPcg's external-exchange path: the operand is
    a host tensor laid out like the library's ([halo below | own | halo
    above], the numpy reference plan); the handle is the numpy test double."""

    def __init__(self, O, sh):
        import torch
        self.O, self.sh = O, sh
        self.dist = types.SimpleNamespace(nccl=False)
        self.x_ext = torch.zeros(sh.n_cols, dtype=torch.float64)
        self.y = torch.zeros(sh.n, dtype=torch.float64)
        self.h = _FakeHandle(O)
        c = sh.csr
        rows = np.repeat(np.arange(sh.n), np.diff(c.row_ptr))
        self.h.diag = np.zeros(sh.n)
        on = c.col == rows + sh.x_offset
        self.h.diag[rows[on]] = c.val[on]

    def own_ptr(self):
        return self.x_ext[self.sh.x_offset:self.sh.x_offset + self.sh.n]

    def set_own(self, x):
        self.own_ptr().copy_(x)


class _FakeExchange:
    """The exchange DistPcg drives (spmv, gather) over gloo, with the halo of
    the numpy reference plan and the oracle's row products."""

    def __init__(self, O, sh):
        import torch.distributed as dist
        self.O, self.sh, self.dist = O, sh, dist
        needs = {q: sh.cols[s:s + c].tolist() for q, (s, c) in sh.recv.items()}
        allneeds = [None] * sh.world
        dist.all_gather_object(allneeds, needs)
        PL.plan_from_needs(sh, {q: allneeds[q][sh.rank] for q in range(sh.world)
                                if q != sh.rank and sh.rank in allneeds[q]})

    def spmv(self, ds, x_own, inject, mode):
        import torch
        dist, sh = self.dist, self.sh
        ops = []
        for q, idx in sorted(sh.send.items()):
            ops.append(dist.P2POp(dist.isend, ds.x_ext[torch.as_tensor(idx)].clone(), q))
        for q, (start, count) in sorted(sh.recv.items()):
            ops.append(dist.P2POp(dist.irecv, ds.x_ext[start:start + count], q))
        if ops:
            for w in dist.batch_isend_irecv(ops):
                w.wait()
        c, xe = sh.csr, ds.x_ext.numpy()
        ds.y.numpy()[:] = [self.O.pw(c.val[c.row_ptr[i]:c.row_ptr[i + 1]] *
                                     xe[c.col[c.row_ptr[i]:c.row_ptr[i + 1]]])
                           for i in range(sh.n)]
        return ds.y

    def gather(self, send, recv):
        self.dist.all_gather_into_tensor(recv, send)


def _gloo_pcg_worker(rank, world, port, variant, q):
    import torch
    import torch.distributed as dist

    from oracle import oracle as O
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = G.laplacian_3d_7pt(8)
        ranges = PL.block_partition(A.n, world, align=64)
        a, b_ = ranges[rank]
        rows = G.stencil_rows("7pt", 8, 8, 8, a // 64, b_ // 64)
        sh = PL.make_shard(rows, a, b_, rank, world, ranges)
        ex = _FakeExchange(O, sh)
        ds = _FakeDs(O, sh)
        p = PL.DistPcg(ds, False, variant)
        bfull = O.spmv(A, G.uniform_vector(A.n, 43))
        b = torch.from_numpy(bfull[a:b_].copy())
        x = torch.from_numpy(G.uniform_vector(A.n, 44)[a:b_].copy())
        hist = []
        state, st = p.solve(ex, b, x, A.n, tol=1e-6, res_hist=hist, poll=4)
        q.put((rank, state, st["iters"], st["spmv_calls"], x.numpy().tolist(), hist))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("variant,world", [("pcg", 2), ("cg1", 2), ("pcg", 3)])
def test_gloo_dist_pcg_protocol(O, variant, world):
    import socket

    import torch.multiprocessing as mp
    A = G.laplacian_3d_7pt(8)
    ranges = PL.block_partition(A.n, world, align=64)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    ref = (O.pcg_cg1_ranks if variant == "cg1" else O.pcg_ranks)(A, b, x0, ranges, tol=1e-6)
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_pcg_worker, args=(r, world, port, variant, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=180) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    x = np.concatenate([np.array(r[4]) for r in res])
    for r in res:
        assert r[1] == 1 and r[2] == ref.iters and r[3] == ref.spmv_calls
        assert np.array_equal(np.array(r[5]), ref.res_hist)
    assert np.array_equal(x.view(np.uint64), ref.x.view(np.uint64))
