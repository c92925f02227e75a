"""Multi-GPU row-block shards through the C ABI (include/abft.h "Multi-GPU"),
on the one GPU this pool has:

* logical ranks in one process, the library's exchange buffers moved by
  LocalExchange (abft_dist_begin -> copies -> abft_dist_end): y, the flags
  of every round and the corrected y bit-exact against the single-GPU oracle,
  error-free and with faults;
* the NCCL communicator path (abft_dist_spmv, abft_dist_pcg) at world 1;
* the distributed PCG (abft_pcg_dist_* phases) against the rank-partitioned
  oracle (R28), fault-free and -- with the union of the ranks' rate-mode
  plans as a per-call oracle fault list -- under faults, bit for bit;
* real processes sharing the GPU over gloo (TorchExchange).
"""
import types

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


def make_dss(A, ranges, **kw):
    from paper_conf_dsn_schollbkw16_b200 import Dist
    rg = PL.ranges_array(ranges)
    dss = []
    for r, (a, b) in enumerate(ranges):
        d = Dist(r, len(ranges), rg)
        dss.append(PL.DistSpmv(d, PL.shard_rows(A, a, b), **kw))
    return dss, PL.LocalExchange(dss)


def local_plan(plan, ranges, r):
    """The entries of a global fault plan that fall on rank r, local indices."""
    a, b = ranges[r]
    sel, idx = [], []
    for e in range(len(plan)):
        t, i = int(plan.target[e]), int(plan.index[e])
        lo, hi = (a, b) if t == 0 else (a // 32, (b + 31) // 32)
        if lo <= i < hi:
            sel.append(e)
            idx.append(i - lo)
    if not sel:
        return None
    return G.FaultPlan(plan.round[sel], plan.target[sel], idx, plan.mask[sel])


def run_sharded(torch, A, ranges, x, plan=None):
    from paper_conf_dsn_schollbkw16_b200 import Inject
    dss, ex = make_dss(A, ranges)
    injects = {}
    for r in range(len(ranges)):
        lp = None if plan is None else local_plan(plan, ranges, r)
        injects[r] = None if lp is None else Inject.from_plan(lp)
    xs = {r: torch.from_numpy(x[a:b].copy()).cuda() for r, (a, b) in enumerate(ranges)}
    ex.spmv_all(xs, injects)
    torch.cuda.synchronize()
    y = np.concatenate([d.y.cpu().numpy() for d in dss])
    flags = [np.sort(np.concatenate([d.h.flags(rnd) + ranges[d.sh.rank][0] // 32 for d in dss]))
             for rnd in range(5)]
    return y, flags, dss


@pytest.mark.parametrize("world", [1, 2, 4])
@pytest.mark.parametrize("name", ["lap3d", "st27", "rand"])
def test_shards_match_oracle(O, torch_cuda, name, world):
    A = {"lap3d": lambda: G.laplacian_3d_7pt(16), "st27": lambda: G.stencil_3d_27pt(12, 12, 16),
         "rand": lambda: G.random_csr(1024, 0.01, 3)}[name]()
    ranges = PL.block_partition(A.n, world)
    x = G.uniform_vector(A.n, 42)
    enc = O.encode(A, 32)
    ref = O.abft_spmv(A, enc, x)
    y, flags, _ = run_sharded(torch_cuda, A, ranges, x)
    assert np.array_equal(y.view(np.uint64), ref.y.view(np.uint64))
    assert flags[0].size == 0
    rng = np.random.default_rng(world)
    idx = rng.choice(A.n, 8, replace=False)
    plan = G.FaultPlan(np.zeros(10), [0] * 8 + [1, 2], list(idx) + [3, enc.nb - 2],
                       [G.burst_mask(int(s), 4) for s in rng.integers(44, 60, 10)])
    ref = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan))
    y, flags, _ = run_sharded(torch_cuda, A, ranges, x, plan)
    for r in range(5):
        assert np.array_equal(flags[r], ref.flags[r]), (r, flags[r], ref.flags[r])
    assert np.array_equal(y.view(np.uint64), ref.y.view(np.uint64))


def test_library_plan_matches_reference_plan(O, torch_cuda):
    """abft_dist_encode's column order, halo slices and send lists equal the
    host reference of parallel.make_shard / exchange_plans."""
    A = G.stencil_3d_27pt(12, 12, 16)
    ranges = PL.block_partition(A.n, 3)
    dss, ex = make_dss(A, ranges)
    shards = [PL.make_shard(PL.shard_rows(A, a, b), a, b, r, 3, ranges)
              for r, (a, b) in enumerate(ranges)]
    PL.exchange_plans(shards, range(3))
    for d, sh in zip(dss, shards):
        assert d.h.n_cols == sh.n_cols and d.h.own_offset == sh.x_offset
        for q in range(3):
            if q == sh.rank:
                continue
            _, sc, _, rc = d.h.buffers(q)
            start, count = sh.recv.get(q, (0, 0))
            assert rc == count
            assert np.array_equal(d.h.needs(q), sh.cols[start:start + count])
            assert sc == len(sh.send.get(q, []))


def test_interior_overlap_split_and_pow2_beta(O, torch_cuda):
    """Large enough for interior chunks: the split changes the launch order,
    never the bits (power-of-two ranges: beta is the single-GPU beta)."""
    A = G.laplacian_3d_7pt(64)
    ranges = PL.block_partition(A.n, 2)
    x = G.uniform_vector(A.n, 5)
    enc = O.encode(A, 32)
    plan = G.FaultPlan([0, 0, 0], [0, 1, 2], [7, 2000, enc.nb - 1], [1 << 62, 1 << 61, 1 << 60])
    ref = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan))
    y, flags, dss = run_sharded(torch_cuda, A, ranges, x, plan)
    assert all(d.h.info()["stream"] == 1 for d in dss)
    for r in range(5):
        assert np.array_equal(flags[r], ref.flags[r])
    assert np.array_equal(y.view(np.uint64), ref.y.view(np.uint64))
    assert dss[0].h.beta() == ref.beta


def test_nccl_world1_spmv_and_pcg(O, torch_cuda):
    """The communicator path (abft_dist_spmv / abft_dist_pcg) at world 1."""
    from paper_conf_dsn_schollbkw16_b200 import Dist, Inject, dist_unique_id
    torch = torch_cuda
    A = G.laplacian_3d_7pt(24)
    d = Dist(0, 1, [0, A.n], dist_unique_id())
    ds = PL.DistSpmv(d, PL.shard_rows(A, 0, A.n))
    x = G.uniform_vector(A.n, 42)
    enc = O.encode(A, 32)
    plan = G.FaultPlan([0, 0], [0, 1], [100, 30], [1 << 62, 1 << 61])
    ref = O.abft_spmv(A, enc, x, O.Inject.from_plan(plan))
    y = ds.spmv(x_own=torch.from_numpy(x).cuda(), inject=Inject.from_plan(plan))
    torch.cuda.synchronize()
    assert np.array_equal(ds.h.flags(0), ref.flags[0])
    assert np.array_equal(y.cpu().numpy().view(np.uint64), ref.y.view(np.uint64))
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    for variant in ("pcg", "cg1"):
        f = O.pcg_cg1_ranks if variant == "cg1" else O.pcg_ranks
        pref = f(A, b, x0, [(0, A.n)], tol=1e-6)
        xd = torch.from_numpy(x0.copy()).cuda()
        hist = torch.zeros(10 * A.n + 1, dtype=torch.float64, device="cuda")
        p = PL.DistPcg(ds, True, variant)
        state, st = p.solve(None, torch.from_numpy(b).cuda(), xd, A.n, tol=1e-6, res_hist=hist)
        assert state == 1 and st["iters"] == pref.iters
        assert np.array_equal(hist[: st["iters"] + 1].cpu().numpy().view(np.uint64),
                              pref.res_hist.view(np.uint64))
        assert np.array_equal(xd.cpu().numpy().view(np.uint64), pref.x.view(np.uint64))


# ---------------------------------------------------------------------------
# Distributed PCG (abft_pcg_dist_*): logical ranks in lockstep on one GPU,
# against the rank-partitioned oracle (R28) bit for bit.
# ---------------------------------------------------------------------------
def run_dist_pcg(torch, A, ranges, b, x0, check=True, tol=1e-6, max_iter=0, variant="pcg",
                 lam=0.0, seed=100):
    from paper_conf_dsn_schollbkw16_b200 import Inject
    dss, ex = make_dss(A, ranges)
    inj = (lambda r: (lambda call: Inject.rate(seed=seed + r, lam=lam, call=call))) if lam else \
        (lambda r: None)
    pcgs = [PL.DistPcg(d, check, variant, inj(d.sh.rank)) for d in dss]
    mi = max_iter if max_iter > 0 else 10 * A.n
    dev = lambda v: torch.from_numpy(np.ascontiguousarray(v)).cuda()  # noqa: E731
    bs = [dev(b[a:b_]) for a, b_ in ranges]
    xs = [dev(x0[a:b_]) for a, b_ in ranges]
    hists = [torch.zeros(mi + 1, dtype=torch.float64, device="cuda") for _ in ranges]
    sts = PL.pcg_lockstep(pcgs, ex, bs, xs, A.n, tol, max_iter, hists)
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


def union_fault_list(O, A, ranges, lam, seed, calls, max_rounds=4):
    """The per-call oracle fault list that equals the ranks' rate-mode plans:
    rank r's plan of SpMV call c (its own ops: rows, local C rows -- the
    library numbers ops per shard) at global indices."""
    enc = O.encode(A, 32)
    rnd, tgt, idx, msk, cll = [], [], [], [], []
    for r, (a, b) in enumerate(ranges):
        rows = PL.shard_rows(A, a, b)
        k0, k1 = a // 32, (b + 31) // 32
        lenc = types.SimpleNamespace(bs=32, row_ptr=np.ascontiguousarray(
            enc.row_ptr[k0:k1 + 1] - enc.row_ptr[k0], dtype=np.int32))
        for c in range(calls):
            ro, ta, ix, mk = O.rate_plan(rows, lenc, O.Inject.rate(seed=seed + r, lam=lam, call=c),
                                         max_rounds)
            rnd += ro.tolist()
            tgt += ta.tolist()
            idx += [int(i) + (a if t == 0 else k0) for i, t in zip(ix, ta)]
            msk += mk.tolist()
            cll += [c] * len(ro)
    return G.FaultPlan(rnd, tgt, idx, np.array(msk, dtype=np.uint64), call=cll)


@pytest.mark.parametrize("world", [2, 4])
def test_dist_pcg_under_faults_bit_exact(O, torch_cuda, world):
    """Rate-mode faults (lambda per arithmetic op) in every rank's
    protected SpMVs (seed 100 + rank, ops numbered per shard) == the
    single-GPU oracle PCG with the union of the ranks' plans as a per-call
    fault list: residual history, solution and flagged-block counts bit for
    bit (equal power-of-two ranges: beta and the dots are the global PW)."""
    A = G.laplacian_3d_7pt(32)
    ranges = [(r * A.n // world, (r + 1) * A.n // world) for r in range(world)]
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    lam = 2e-6
    st, x, hist, sts = run_dist_pcg(torch_cuda, A, ranges, b, x0, True, lam=lam)
    calls = sts[0][1]["spmv_calls"]
    plan = union_fault_list(O, A, ranges, lam, 100, calls)
    assert len(plan) > 0
    enc = O.encode(A, 32)
    ref = O.pcg(A, enc, b, x0, tol=1e-6, inj=O.Inject.from_plan(plan))
    assert st == 1 and ref.status == 0
    assert sts[0][1]["iters"] == ref.iters and calls == ref.spmv_calls
    assert sum(s[1]["flagged_blocks"] for s in sts) == ref.flagged_blocks > 0
    assert np.array_equal(hist.view(np.uint64), ref.res_hist.view(np.uint64))
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


def _dist_pcg_worker(rank, world, port, outdir, variant="pcg"):
    """One process per rank on the same GPU (gloo process group; the NCCL
    communicator needs one GPU per rank): the library's exchange buffers moved
    by TorchExchange."""
    import os

    import torch
    import torch.distributed as dist

    from paper_conf_dsn_schollbkw16_b200 import Dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    n3 = 24
    A = G.laplacian_3d_7pt(n3)
    ranges = PL.block_partition(A.n, world, align=n3 * n3)
    a, b_ = ranges[rank]
    rows = G.stencil_rows("7pt", n3, n3, n3, a // (n3 * n3), b_ // (n3 * n3))
    d = PL.DistSpmv(Dist(rank, world, PL.ranges_array(ranges)), rows)
    ex = PL.TorchExchange(d)
    bfull = np.load(os.path.join(outdir, "b.npy"))
    x0 = np.load(os.path.join(outdir, "x0.npy"))
    b = torch.from_numpy(bfull[a:b_].copy()).cuda()
    x = torch.from_numpy(x0[a:b_].copy()).cuda()
    hist = torch.zeros(10 * A.n + 1, dtype=torch.float64, device="cuda")
    state, st = PL.DistPcg(d, True, variant).solve(ex, b, x, A.n, tol=1e-6, res_hist=hist)
    torch.cuda.synchronize()
    np.save(os.path.join(outdir, f"x{rank}.npy"), x.cpu().numpy())
    np.save(os.path.join(outdir, f"h{rank}.npy"), hist[: st["iters"] + 1].cpu().numpy())
    np.save(os.path.join(outdir, f"s{rank}.npy"), np.array([state, st["iters"]]))
    dist.destroy_process_group()


@pytest.mark.parametrize("world,variant", [(2, "pcg"), (3, "pcg"), (2, "cg1")])
def test_dist_pcg_processes(O, torch_cuda, tmp_path, world, variant):
    """DistPcg.solve across real processes (library buffers, gloo staging
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


@pytest.mark.parametrize("eager", [False, True])
@pytest.mark.parametrize("variant", ["pcg", "cg1"])
def test_nccl_world1_pcg_graph_and_eager(O, torch_cuda, variant, eager, monkeypatch):
    """abft_dist_pcg replays a captured 16-iteration graph for fault-free
    solves (ABFT_DIST_PCG_EAGER=1: eager sequencing); both give the oracle's
    bits, a second solve on the same buffers reuses the cached graph, and a
    max_iter that is not a multiple of 16 stops exactly there."""
    from paper_conf_dsn_schollbkw16_b200 import Dist, dist_unique_id
    torch = torch_cuda
    if eager:
        monkeypatch.setenv("ABFT_DIST_PCG_EAGER", "1")
    A = G.laplacian_3d_7pt(20)
    d = Dist(0, 1, [0, A.n], dist_unique_id())
    ds = PL.DistSpmv(d, PL.shard_rows(A, 0, A.n))
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    f = O.pcg_cg1_ranks if variant == "cg1" else O.pcg_ranks
    for max_iter in (0, 0, 21):
        pref = f(A, b, x0, [(0, A.n)], tol=1e-6, max_iter=max_iter)
        xd = torch.from_numpy(x0.copy()).cuda()
        hist = torch.zeros(10 * A.n + 1, dtype=torch.float64, device="cuda")
        p = PL.DistPcg(ds, True, variant)
        state, st = p.solve(None, torch.from_numpy(b).cuda(), xd, A.n, tol=1e-6,
                            max_iter=max_iter, res_hist=hist)
        assert st["iters"] == pref.iters, (max_iter, st["iters"], pref.iters)
        assert state == (1 if max_iter == 0 else 3), state
        assert np.array_equal(hist[: st["iters"] + 1].cpu().numpy().view(np.uint64),
                              pref.res_hist.view(np.uint64))
        assert np.array_equal(xd.cpu().numpy().view(np.uint64), pref.x.view(np.uint64))
