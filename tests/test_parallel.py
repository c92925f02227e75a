"""Row-block sharding -- host logic on CPU.

* in-process: every shard's local (global-order) CSR, its halo and the
  oracle's SpMV / encoding on it reproduce the global oracle bit for bit;
  the PW of the per-rank x^2 partials equals the global one;
* 2 processes over gloo: the halo exchange and the partial all-gather.
"""
import os

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


def _gloo_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = G.laplacian_3d_7pt(8)
        x = G.uniform_vector(A.n, 42)
        ranges = PL.block_partition(A.n, world)
        a, b = ranges[rank]
        rows = G.CSR(A.row_ptr[a:b + 1] - A.row_ptr[a], A.col[A.row_ptr[a]:A.row_ptr[b]],
                     A.val[A.row_ptr[a]:A.row_ptr[b]])
        sh = PL.make_shard(rows, a, b, rank, world, ranges)
        comm = PL.TorchDistComm()
        PL.plan_from_needs(sh, comm.gather_needs(sh))
        ext = torch.zeros(sh.n_cols, dtype=torch.float64)
        ext[sh.x_offset:sh.x_offset + sh.n] = torch.from_numpy(x[a:b])
        comm.halo(sh, ext)
        ok = bool(np.array_equal(ext.numpy(), x[sh.cols]))
        part = torch.tensor([float(rank + 1)], dtype=torch.float64)
        out = torch.empty(world, dtype=torch.float64)
        comm.gather_partials(part, out)
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
