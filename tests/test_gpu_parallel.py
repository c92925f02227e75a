"""Row-block shards on one GPU (logical ranks, in-process halo copies): the
distributed protected SpMV path of the C ABI (rectangular shard matrices,
ABFT_DEFER_FINISH, abft_beta_partial, abft_finish) must reproduce the
single-handle run and the oracle bit for bit -- y, flags per round and the
corrected y."""
import numpy as np
import pytest

from paper_conf_dsn_schollbkw16_b200 import inputs as G
from paper_conf_dsn_schollbkw16_b200 import parallel as PL

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required")
    from paper_conf_dsn_schollbkw16_b200 import _build
    _build.build()
    return torch


def run_sharded(torch, A, world, x, plan=None):
    from paper_conf_dsn_schollbkw16_b200 import Inject
    ranges = PL.block_partition(A.n, world)
    shards = []
    for r, (a, b) in enumerate(ranges):
        rows = G.CSR(A.row_ptr[a:b + 1] - A.row_ptr[a], A.col[A.row_ptr[a]:A.row_ptr[b]],
                     A.val[A.row_ptr[a]:A.row_ptr[b]])
        shards.append(PL.make_shard(rows, a, b, r, world, ranges))
    PL.exchange_plans(shards, range(world))
    ds = [PL.DistSpmv(sh) for sh in shards]
    for d, sh in zip(ds, shards):
        d.own().copy_(torch.from_numpy(x[sh.row0:sh.row1]))
    comm = PL.LocalComm(shards, {d.sh.rank: d.x_ext for d in ds})
    injs = []
    for sh in shards:
        inj = None
        if plan is not None:
            sel, idx = [], []
            for e in range(len(plan)):
                t, i = int(plan.target[e]), int(plan.index[e])
                lo, hi = (sh.row0, sh.row1) if t == 0 else (sh.row0 // 32, (sh.row1 + 31) // 32)
                if lo <= i < hi:
                    sel.append(e)
                    idx.append(i - lo)
            if sel:
                inj = Inject.from_plan(G.FaultPlan(plan.round[sel], plan.target[sel], idx,
                                                   plan.mask[sel]))
        injs.append(inj)
    parts = []
    for d, inj in zip(ds, injs):
        parts.append(d.step1(comm, inj))
    allp = torch.cat(parts)
    for d, inj in zip(ds, injs):
        d.parts.copy_(allp)
        d.step2(None, inj)
    torch.cuda.synchronize()
    y = np.concatenate([d.y.cpu().numpy() for d in ds])
    flags = []
    for rnd in range(5):
        f = [d.h.flags(rnd) + d.sh.row0 // 32 for d in ds]
        flags.append(np.sort(np.concatenate(f)))
    return y, flags


@pytest.mark.parametrize("world", [1, 2, 4])
@pytest.mark.parametrize("name", ["lap3d", "st27", "rand"])
def test_shards_match_oracle(O, torch_cuda, name, world):
    A = {"lap3d": lambda: G.laplacian_3d_7pt(16), "st27": lambda: G.stencil_3d_27pt(12, 12, 16),
         "rand": lambda: G.random_csr(1024, 0.01, 3)}[name]()
    x = G.uniform_vector(A.n, 42)
    enc = O.encode(A, 32)
    ref = O.abft_spmv(A, enc, x)
    y, flags = run_sharded(torch_cuda, A, world, x)
    assert np.array_equal(y.view(np.uint64), ref.y.view(np.uint64))
    assert flags[0].size == 0
    rng = np.random.default_rng(world)
    idx = rng.choice(A.n, 8, replace=False)
    plan = G.FaultPlan(np.zeros(10), [0] * 8 + [1, 2], list(idx) + [3, enc.nb - 2],
                       [G.burst_mask(int(s), 4) for s in rng.integers(44, 60, 10)])
    ref = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan))
    y, flags = run_sharded(torch_cuda, A, world, x, plan)
    for r in range(5):
        assert np.array_equal(flags[r], ref.flags[r]), (r, flags[r], ref.flags[r])
    assert np.array_equal(y.view(np.uint64), ref.y.view(np.uint64))
