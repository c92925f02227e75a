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


# ---------------------------------------------------------------------------
# Distributed PCG (abft_pcg_dist_*): logical ranks in lockstep on one GPU,
# against the rank-partitioned oracle (R28) bit for bit.
# ---------------------------------------------------------------------------
def make_shards(A, ranges):
    world = len(ranges)
    shards = []
    for r, (a, b) in enumerate(ranges):
        rows = G.CSR(A.row_ptr[a:b + 1] - A.row_ptr[a], A.col[A.row_ptr[a]:A.row_ptr[b]],
                     A.val[A.row_ptr[a]:A.row_ptr[b]])
        shards.append(PL.make_shard(rows, a, b, r, world, ranges))
    PL.exchange_plans(shards, range(world))
    return shards


def run_dist_pcg(torch, A, ranges, b, x0, check=True, tol=1e-6, max_iter=0, variant="pcg",
                 lam=0.0, graph=False):
    shards = make_shards(A, ranges)
    ds = [PL.DistSpmv(sh) for sh in shards]
    comm = PL.LocalComm(shards, {d.sh.rank: d.x_ext for d in ds})
    from paper_conf_dsn_schollbkw16_b200 import Inject
    inj = (lambda r: (lambda call: Inject.rate(seed=100 + r, lam=lam, call=call))) if lam else \
        (lambda r: None)
    pcgs = [PL.DistPcg(d, check, variant, inj(d.sh.rank)) for d in ds]
    mi = max_iter if max_iter > 0 else 10 * A.n
    dev = lambda v: torch.from_numpy(np.ascontiguousarray(v)).cuda()
    bs = [dev(b[sh.row0:sh.row1]) for sh in shards]
    xs = [dev(x0[sh.row0:sh.row1]) for sh in shards]
    hists = [torch.zeros(mi + 1, dtype=torch.float64, device="cuda") for _ in shards]
    sts = PL.pcg_lockstep(pcgs, comm, bs, xs, A.n, tol, max_iter, hists, graph=graph)
    torch.cuda.synchronize()
    x = np.concatenate([v.cpu().numpy() for v in xs])
    it = sts[0][1]["iters"]
    for s in sts:  # every rank holds the same scalars
        assert s[0] == sts[0][0] and s[1]["iters"] == it
        assert s[1]["final_residual"] == sts[0][1]["final_residual"]
    return sts[0][0], x, hists[0][: it + 1].cpu().numpy(), sts


@pytest.mark.parametrize("check", [True, False])
@pytest.mark.parametrize("case", ["pow2-2", "pow2-4", "planes-3", "st27-3", "ragged-2"])
def test_dist_pcg_matches_oracle(O, torch_cuda, case, check):
    if case.startswith("pow2"):
        A = G.laplacian_3d_7pt(32)  # 32768 rows: ranks of 16384 / 8192 (aligned)
        w = int(case[-1])
        ranges = [(r * A.n // w, (r + 1) * A.n // w) for r in range(w)]
    elif case == "planes-3":
        A = G.laplacian_3d_7pt(24)  # 8 planes per rank, not powers of two
        ranges = [(0, 4608), (4608, 9216), (9216, A.n)]
    elif case == "st27-3":
        A = G.stencil_3d_27pt(20, 20, 24)  # odd halo widths: unaligned own slices
        ranges = PL.block_partition(A.n, 3)
    else:
        A = G.laplacian_3d_7pt(21)  # 9261 rows, ragged last block
        ranges = PL.block_partition(A.n, 2)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    ref = O.pcg_ranks(A, b, x0, ranges, tol=1e-6)
    assert ref.status == 0
    st, x, hist, sts = run_dist_pcg(torch_cuda, A, ranges, b, x0, check)
    assert st == 1  # converged
    assert sts[0][1]["iters"] == ref.iters
    assert np.array_equal(hist.view(np.uint64), ref.res_hist.view(np.uint64))
    assert np.array_equal(x.view(np.uint64), ref.x.view(np.uint64))
    calls = sum(s[1]["spmv_calls"] for s in sts) // len(sts)
    assert calls == ref.spmv_calls
    if check:
        assert all(s[1]["uncorrected_calls"] == 0 for s in sts)


def test_dist_pcg_pow2_equals_single_gpu(O, torch_cuda):
    """Equal power-of-two ranges: the distributed solve is the single-GPU
    abft_pcg bit for bit (R2 padding independence)."""
    from paper_conf_dsn_schollbkw16_b200 import abft
    torch = torch_cuda
    A = G.laplacian_3d_7pt(32)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    h = abft.encode(A)
    xd = torch.from_numpy(x0.copy()).cuda()
    hist1 = torch.zeros(10 * A.n + 1, dtype=torch.float64, device="cuda")
    status, st1 = h.pcg(torch.from_numpy(b).cuda(), xd, tol=1e-6, res_hist=hist1)
    ranges = [(r * A.n // 4, (r + 1) * A.n // 4) for r in range(4)]
    st, x, hist, sts = run_dist_pcg(torch, A, ranges, b, x0)
    assert st1["iters"] == sts[0][1]["iters"]
    assert np.array_equal(x.view(np.uint64), xd.cpu().numpy().view(np.uint64))
    assert np.array_equal(hist.view(np.uint64),
                          hist1[: st1["iters"] + 1].cpu().numpy().view(np.uint64))


def _dist_pcg_worker(rank, world, port, outdir, variant="pcg"):
    """One process per rank on the same GPU (gloo process group: the NCCL
    path needs one GPU per rank): DistPcg.solve with TorchDistComm."""
    import os

    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    n3 = 24
    A = G.laplacian_3d_7pt(n3)
    ranges = PL.block_partition(A.n, world, align=n3 * n3)
    a, b_ = ranges[rank]
    rows = G.stencil_rows("7pt", n3, n3, n3, a // (n3 * n3), b_ // (n3 * n3))
    sh = PL.make_shard(rows, a, b_, rank, world, ranges)
    comm = PL.TorchDistComm()
    PL.plan_from_needs(sh, comm.gather_needs(sh))
    d = PL.DistSpmv(sh)
    bfull = np.load(os.path.join(outdir, "b.npy"))
    x0 = np.load(os.path.join(outdir, "x0.npy"))
    b = torch.from_numpy(bfull[a:b_].copy()).cuda()
    x = torch.from_numpy(x0[a:b_].copy()).cuda()
    hist = torch.zeros(10 * A.n + 1, dtype=torch.float64, device="cuda")
    state, st = PL.DistPcg(d, True, variant).solve(comm, b, x, A.n, tol=1e-6, res_hist=hist)
    torch.cuda.synchronize()
    np.save(os.path.join(outdir, f"x{rank}.npy"), x.cpu().numpy())
    np.save(os.path.join(outdir, f"h{rank}.npy"), hist[: st["iters"] + 1].cpu().numpy())
    np.save(os.path.join(outdir, f"s{rank}.npy"), np.array([state, st["iters"]]))
    dist.destroy_process_group()


@pytest.mark.parametrize("world,variant", [(2, "pcg"), (3, "pcg"), (2, "cg1")])
def test_dist_pcg_processes(O, torch_cuda, tmp_path, world, variant):
    """DistPcg.solve across real processes (torch.distributed, gloo staging
    through the host) == the rank-partitioned oracle bit for bit."""
    import socket

    import torch.multiprocessing as mp
    n3 = 24
    A = G.laplacian_3d_7pt(n3)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    np.save(tmp_path / "b.npy", b)
    np.save(tmp_path / "x0.npy", x0)
    ranges = PL.block_partition(A.n, world, align=n3 * n3)
    ref = (O.pcg_cg1_ranks if variant == "cg1" else O.pcg_ranks)(A, b, x0, ranges, tol=1e-6)
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    mp.start_processes(_dist_pcg_worker, args=(world, port, str(tmp_path), variant), nprocs=world,
                       join=True, start_method="spawn")
    x = np.concatenate([np.load(tmp_path / f"x{r}.npy") for r in range(world)])
    for r in range(world):
        state, it = np.load(tmp_path / f"s{r}.npy")
        assert state == 1 and it == ref.iters
        assert np.array_equal(np.load(tmp_path / f"h{r}.npy").view(np.uint64),
                              ref.res_hist.view(np.uint64))
    assert np.array_equal(x.view(np.uint64), ref.x.view(np.uint64))


@pytest.mark.parametrize("check", [True, False])
@pytest.mark.parametrize("case", ["1", "pow2-4", "planes-3", "st27-3", "ragged-2"])
def test_dist_cg1_matches_oracle(O, torch_cuda, case, check):
    """Single-reduction PCG (R29) == oracle pcg_cg1_ranks bit for bit."""
    if case == "1":
        A = G.laplacian_3d_7pt(20)
        ranges = [(0, A.n)]
    elif case == "pow2-4":
        A = G.laplacian_3d_7pt(32)
        ranges = [(r * A.n // 4, (r + 1) * A.n // 4) for r in range(4)]
    elif case == "planes-3":
        A = G.laplacian_3d_7pt(24)
        ranges = [(0, 4608), (4608, 9216), (9216, A.n)]
    elif case == "st27-3":
        A = G.stencil_3d_27pt(20, 20, 24)
        ranges = PL.block_partition(A.n, 3)
    else:
        A = G.laplacian_3d_7pt(21)
        ranges = PL.block_partition(A.n, 2)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    ref = O.pcg_cg1_ranks(A, b, x0, ranges, tol=1e-6)
    assert ref.status == 0
    st, x, hist, sts = run_dist_pcg(torch_cuda, A, ranges, b, x0, check, variant="cg1")
    assert st == 1
    assert sts[0][1]["iters"] == ref.iters
    assert sts[0][1]["spmv_calls"] == ref.spmv_calls
    assert np.array_equal(hist.view(np.uint64), ref.res_hist.view(np.uint64))
    assert np.array_equal(x.view(np.uint64), ref.x.view(np.uint64))


def test_dist_cg1_maxiter(O, torch_cuda):
    A = G.laplacian_3d_7pt(16)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    ranges = PL.block_partition(A.n, 2)
    ref = O.pcg_cg1_ranks(A, b, x0, ranges, tol=1e-6, max_iter=5)
    st, x, hist, sts = run_dist_pcg(torch_cuda, A, ranges, b, x0, True, max_iter=5,
                                    variant="cg1")
    assert ref.status == -5 and st == 3 and sts[0][1]["iters"] == ref.iters == 5
    assert np.array_equal(hist.view(np.uint64), ref.res_hist.view(np.uint64))
    assert np.array_equal(x.view(np.uint64), ref.x.view(np.uint64))


@pytest.mark.parametrize("variant", ["pcg", "cg1"])
def test_dist_pcg_under_faults(O, torch_cuda, variant):
    """Rate-mode faults (lambda per arithmetic op) in every rank's
    protected SpMVs: the solve still converges, faults are flagged and
    corrected (none left uncorrected), and the solution solves A x = b."""
    A = G.laplacian_3d_7pt(24)
    ranges = [(0, 4608), (4608, 9216), (9216, A.n)]
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    st, x, hist, sts = run_dist_pcg(torch_cuda, A, ranges, b, x0, True, variant=variant,
                                    lam=1e-5)
    assert st == 1
    assert sum(s[1]["flagged_blocks"] for s in sts) > 0
    assert all(s[1]["uncorrected_calls"] == 0 for s in sts)
    ref = (O.pcg_cg1_ranks if variant == "cg1" else O.pcg_ranks)(A, b, x0, ranges, tol=1e-6)
    assert abs(sts[0][1]["iters"] - ref.iters) <= 2
    rel = np.linalg.norm(b - O.spmv(A, x)) / np.linalg.norm(b)
    assert rel <= 1e-5


@pytest.mark.parametrize("variant", ["pcg", "cg1"])
@pytest.mark.parametrize("check", [True, False])
def test_dist_pcg_graph_replay(O, torch_cuda, variant, check):
    """CUDA-graph replay of 16-iteration batches == the oracle bit for bit
    (2 logical ranks; max_iter not a multiple of the batch: the tail runs
    eagerly)."""
    A = G.laplacian_3d_7pt(24)
    ranges = PL.block_partition(A.n, 2)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    f = O.pcg_cg1_ranks if variant == "cg1" else O.pcg_ranks
    for mi in (0, 37):
        ref = f(A, b, x0, ranges, tol=1e-6, max_iter=mi)
        st, x, hist, sts = run_dist_pcg(torch_cuda, A, ranges, b, x0, check, max_iter=mi,
                                        variant=variant, graph=True)
        assert sts[0][1]["iters"] == ref.iters
        assert np.array_equal(hist.view(np.uint64), ref.res_hist.view(np.uint64))
        assert np.array_equal(x.view(np.uint64), ref.x.view(np.uint64))


def test_dist_pcg_graph_reuse(O, torch_cuda):
    """A second solve on the same buffers replays the cached graph and gives
    the same bits (x reset to x0 between solves)."""
    torch = torch_cuda
    A = G.laplacian_3d_7pt(20)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    ref = O.pcg_ranks(A, b, x0, [(0, A.n)], tol=1e-6)
    (sh,) = make_shards(A, [(0, A.n)])
    d = PL.DistSpmv(sh)
    p = PL.DistPcg(d, True)

    class Solo:
        def gather_partials(self, part, out):
            out.copy_(part)

        def halo(self, s_, x_ext):
            pass

    bd = torch.from_numpy(b).cuda()
    xd = torch.empty(A.n, dtype=torch.float64, device="cuda")
    for rep in range(3):
        xd.copy_(torch.from_numpy(x0))
        state, st = p.solve(Solo(), bd, xd, A.n, tol=1e-6, graph=True)
        torch.cuda.synchronize()
        assert state == 1 and st["iters"] == ref.iters
        assert np.array_equal(xd.cpu().numpy().view(np.uint64), ref.x.view(np.uint64))
    assert p._graph is not None
