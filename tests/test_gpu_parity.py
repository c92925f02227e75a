"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on
the same seeded inputs and the same fault plans.

Bar (BASELINE.json north_star): flagged-block sets and corrected-block
indices bit-exact; corrected y within 1e-12 relative (we require -- and get --
bit-exact y, t1, t2, beta, C and K because both sides follow the same PW
order, R2); PCG residual histories within 1e-10 relative (again we
assert bit-exact and keep the 1e-10 check as the stated bar).
"""
import numpy as np
import pytest

from paper_conf_dsn_schollbkw16_b200 import inputs as G

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    from paper_conf_dsn_schollbkw16_b200 import _build
    _build.build()
    return torch


def bits(a):
    return np.ascontiguousarray(a, dtype=np.float64).view(np.uint64)


def assert_bits_equal(a, b, what):
    a, b = bits(a), bits(b)
    if not np.array_equal(a, b):
        bad = np.nonzero(a != b)[0]
        raise AssertionError(f"{what}: {bad.size} mismatches, first at {bad[:5].tolist()}: "
                             f"{a.view(np.float64)[bad[:3]]} vs {b.view(np.float64)[bad[:3]]}")


def oracle_inject(O, plan=None, rate=None):
    if plan is not None:
        return O.Inject.from_plan(plan)
    if rate is not None:
        return O.Inject.rate(**rate)
    return None


def gpu_inject(plan=None, rate=None):
    from paper_conf_dsn_schollbkw16_b200 import Inject
    if plan is not None:
        return Inject.from_plan(plan)
    if rate is not None:
        return Inject.rate(**rate)
    return None


class Case:
    """Encode A on both sides once; run protected SpMVs on both."""

    def __init__(self, O, torch, A, bs=32, max_rounds=4, c_csr=False):
        from paper_conf_dsn_schollbkw16_b200 import encode
        self.O, self.torch, self.A, self.bs = O, torch, A, bs
        self.enc = O.encode(A, bs)
        self.h = encode(A, bs, max_rounds, c_csr=c_csr)
        self.max_rounds = max_rounds

    def check_encoding(self):
        rp, col, val, K = self.h.checksum_matrix()
        assert np.array_equal(rp, self.enc.row_ptr)
        assert np.array_equal(col, self.enc.col)
        assert_bits_equal(val, self.enc.val, "C values")
        assert_bits_equal(K, self.enc.K, "K")

    def run(self, x, plan=None, rate=None, x_norm=False):
        from paper_conf_dsn_schollbkw16_b200 import CHECK, DEBUG_CHECKSUMS
        torch = self.torch
        ref = self.O.abft_spmv(self.A, self.enc, x, oracle_inject(self.O, plan, rate),
                               self.max_rounds)
        xd = torch.from_numpy(x).cuda()
        xn = torch.tensor([ref.beta], dtype=torch.float64, device="cuda") if x_norm else None
        inj = gpu_inject(plan, rate)
        y = self.h.spmv(xd, x_norm=xn, inject=inj, mode=CHECK | DEBUG_CHECKSUMS)
        torch.cuda.synchronize()
        assert_bits_equal(y.cpu().numpy(), ref.y_pre, "y (pre-correction)")
        t1, t2 = self.h.debug_checksums()
        # the oracle's t1/t2 hold the last round's values for recomputed blocks
        keep = np.ones(self.enc.nb, dtype=bool)
        for f in ref.flags[:-1]:
            keep[f] = False
        assert_bits_equal(t1[keep], ref.t1[keep], "t1")
        assert_bits_equal(t2[keep], ref.t2[keep], "t2")
        assert self.h.beta() == ref.beta
        assert np.array_equal(self.h.flags(0), ref.flags[0]), (self.h.flags(0), ref.flags[0])
        self.h.correct(xd, y, self.max_rounds, inject=inj)
        torch.cuda.synchronize()
        for r in range(1, self.max_rounds + 1):
            assert np.array_equal(self.h.flags(r), ref.flags[r]), (r, self.h.flags(r), ref.flags[r])
        assert_bits_equal(y.cpu().numpy(), ref.y, "y (corrected)")
        return ref


def _mixed_lean_irr():
    """Mostly short rows (k_lean majority) with a few groups holding rows of
    33..600 entries (k_irr) and one hub row > 1024 entries (k_general)."""
    rng = np.random.Generator(np.random.PCG64(17))
    n = 4096
    lens = rng.integers(0, 9, n)
    lens[[70, 1000, 1001, 2050, 3333]] = [40, 300, 600, 33, 129]
    lens[3900] = 1500
    rows, cols = [], []
    for i, L in enumerate(lens):
        c = np.sort(rng.choice(n, size=int(L), replace=False))
        rows.append(np.full(c.size, i))
        cols.append(c)
    cols = np.concatenate(cols).astype(np.int32)
    rp = np.zeros(n + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    return G.CSR(rp.astype(np.int32), cols, rng.uniform(-1, 1, cols.size), "mixed_lean_irr")


MATRICES = {
    "lap2d_64": lambda: G.laplacian_2d_5pt(64),           # BASELINE configs[0]
    "lap3d_16": lambda: G.laplacian_3d_7pt(16),
    "lap3d_ragged": lambda: G.laplacian_3d_7pt(13, 11, 7),  # 1001 rows: ragged tail
    "st27_11": lambda: G.stencil_3d_27pt(11),               # 27-pt, 1331 rows
    "rand_empty": lambda: G.random_csr(1000, 0.01, 3, empty_rows=0.2),
    "rand_dense": lambda: G.random_csr(300, 0.3, 4),        # rows > 32: warp fallback
    "rmat11": lambda: G.rmat(11, 16, 5),                    # power law, long rows
    "rmat11_natural": lambda: G.rmat(11, 8, 6, permute=False),  # empty blocks
    "hubs": lambda: G.hub_csr(5000, 11),                    # rows / C rows > 1024: hub chunks
    "mixed_lean_irr": lambda: _mixed_lean_irr(),            # k_lean + k_irr + k_general
    "tiny1": lambda: G.CSR([0, 1], [0], [2.5]),
    "tiny33": lambda: G.random_csr(33, 0.2, 9),
    "all_empty": lambda: G.CSR(np.zeros(101, np.int32), np.zeros(0, np.int32), np.zeros(0)),
}


@pytest.mark.parametrize("c_csr", [False, True])
@pytest.mark.parametrize("name", sorted(MATRICES))
def test_encode_and_spmv_error_free(O, torch_cuda, name, c_csr):
    A = MATRICES[name]()
    c = Case(O, torch_cuda, A, c_csr=c_csr)
    c.check_encoding()
    for seed in (42, 43):
        ref = c.run(G.uniform_vector(A.n, seed))
        assert ref.flagged.size == 0


@pytest.mark.parametrize("bs", [1, 2, 4, 8, 16])
@pytest.mark.parametrize("name", ["lap3d_ragged", "rmat11", "rand_dense", "hubs"])
def test_block_sizes(O, torch_cuda, name, bs):
    A = MATRICES[name]()
    c = Case(O, torch_cuda, A, bs=bs)
    c.check_encoding()
    c.run(G.uniform_vector(A.n, 7))
    plan = G.FaultPlan([0, 0, 0], [0, 1, 2], [A.n // 2, 1, c.enc.nb - 1], [1 << 62, 1 << 61, 1 << 60])
    ref = c.run(G.uniform_vector(A.n, 8), plan=plan)
    assert ref.flagged.size >= 1


@pytest.mark.parametrize("c_csr", [False, True])
def test_hub_rows_faults(O, torch_cuda, c_csr):
    """Faults in hub rows (> 1024 entries, chunked by k_hub) and in the
    checksums of blocks whose C row is a hub: flagged, localized, corrected."""
    A = MATRICES["hubs"]()
    c = Case(O, torch_cuda, A, c_csr=c_csr)
    hub_rows = np.nonzero(np.diff(A.row_ptr) > 1024)[0]
    assert hub_rows.size >= 2
    kb = int(hub_rows[1]) // 32
    plan = G.FaultPlan([0, 0, 0, 1], [0, 0, 1, 0], [int(hub_rows[0]), int(hub_rows[1]) , kb, 5],
                       [1 << 62, 1 << 55, 1 << 60, 1 << 61])
    ref = c.run(G.uniform_vector(A.n, 21), plan=plan)
    assert set(ref.flags[0].tolist()) >= {int(hub_rows[0]) // 32, kb}


def test_single_bit_flips_config0(O, torch_cuda):
    # BASELINE configs[0]: 64x64 5-pt, one seeded burst per run.
    A = MATRICES["lap2d_64"]()
    c = Case(O, torch_cuda, A)
    x = G.uniform_vector(A.n, 42)
    detected = 0
    for seed in range(60):
        plan = G.single_fault_plan(A.n, seed)
        ref = c.run(x, plan=plan)
        detected += ref.flagged.size
    assert detected > 30


@pytest.mark.parametrize("c_csr", [False, True])
@pytest.mark.parametrize("target", [0, 1, 2])
def test_checksum_and_result_targets(O, torch_cuda, target, c_csr):
    A = MATRICES["st27_11"]()
    c = Case(O, torch_cuda, A, c_csr=c_csr)
    n_el = A.n if target == 0 else c.enc.nb
    rng = np.random.default_rng(target)
    idx = rng.choice(n_el, 12, replace=False)
    plan = G.FaultPlan(np.zeros(12), np.full(12, target), idx,
                       [G.burst_mask(int(s), 3) for s in rng.integers(40, 61, 12)])
    ref = c.run(G.uniform_vector(A.n, 5), plan=plan)
    assert ref.flagged.size > 0


def test_faults_in_correction_rounds(O, torch_cuda):
    # faults injected into the recomputation itself (rounds 1, 2): the block
    # stays flagged for those rounds; round 4 exhausts -> uncorrected set.
    A = MATRICES["lap3d_16"]()
    c = Case(O, torch_cuda, A)
    k = 17
    i = k * 32 + 3
    plan = G.FaultPlan([0, 1, 2, 1, 2, 3, 4], [0, 0, 2, 0, 1, 0, 0],
                       [i, i, k, 100 * 32, k, i, i],
                       [1 << 62, 1 << 62, 1 << 62, 1 << 62, 1 << 55, 1 << 62, 1 << 62])
    ref = c.run(G.uniform_vector(A.n, 3), plan=plan)
    assert ref.flags[4].tolist() == [k] and ref.status == -6


@pytest.mark.parametrize("lam", [1e-6, 1e-4, 1e-2])
def test_rate_mode(O, torch_cuda, lam):
    # P:284 rate model through the device-side Philox injector.
    A = MATRICES["lap3d_16"]()
    c = Case(O, torch_cuda, A)
    for call in range(3):
        c.run(G.uniform_vector(A.n, 11 + call), rate=dict(seed=99, lam=lam, targets=0b111, call=call))


def test_rate_mode_rmat_bs8(O, torch_cuda):
    A = MATRICES["rmat11"]()
    c = Case(O, torch_cuda, A, bs=8)
    c.run(G.uniform_vector(A.n, 1), rate=dict(seed=5, lam=1e-3, targets=0b111, call=7))


def test_compact_formats_chosen(O, torch_cuda, monkeypatch):
    # the encoder picks the narrowest exact type; row-
    # regular matrices get position-map records (§6.9), the others the slot map
    from paper_conf_dsn_schollbkw16_b200 import encode
    cases = [(G.laplacian_3d_7pt(16), "int8+pos"), (G.random_csr(500, 0.02, 1), "f64+u16"),
             (G.random_csr(300, 0.05, 2, integer=True, max_int=100), "int16+u16")]
    for A, fmt in cases:
        info = encode(A).info()
        assert info["c_format_name"] == fmt, (A.name, info)
    info = encode(G.laplacian_3d_7pt(16), c_csr=True).info()
    assert info["c_format_name"] == "csr-f64"
    A = G.laplacian_3d_7pt(16)
    info = encode(A).info()
    assert info["general_groups"] == 0 and info["stream"] == 1
    monkeypatch.setenv("ABFT_NO_POS", "1")
    info = encode(A).info()
    assert info["c_format_name"] == "int8+u16"
    assert info["general_groups"] == 0 and info["lean"] == 1


@pytest.mark.parametrize("lam", [1e-4])
def test_rate_mode_csr_c(O, torch_cuda, lam):
    A = MATRICES["lap3d_16"]()
    c = Case(O, torch_cuda, A, c_csr=True)
    c.run(G.uniform_vector(A.n, 11), rate=dict(seed=99, lam=lam, targets=0b111, call=5))


def test_x_norm_given(O, torch_cuda):
    A = MATRICES["lap3d_16"]()
    c = Case(O, torch_cuda, A)
    plan = G.single_fault_plan(A.n, 3)
    c.run(G.uniform_vector(A.n, 42), plan=plan, x_norm=True)


def test_nan_and_zero(O, torch_cuda):
    A = MATRICES["lap3d_ragged"]()
    c = Case(O, torch_cuda, A)
    c.run(np.zeros(A.n))
    plan = G.FaultPlan([0], [0], [A.n - 1], [0x7FF8000000000000])
    ref = c.run(G.uniform_vector(A.n, 1), plan=plan)
    assert ref.flagged.tolist() == [(A.n - 1) // 32]


def test_repeated_calls_reset_state(O, torch_cuda):
    from paper_conf_dsn_schollbkw16_b200 import CHECK
    A = MATRICES["lap2d_64"]()
    c = Case(O, torch_cuda, A)
    x = torch_cuda.from_numpy(G.uniform_vector(A.n, 1)).cuda()
    inj = gpu_inject(plan=G.FaultPlan([0], [0], [5], [1 << 62]))
    c.h.spmv(x, inject=inj, mode=CHECK)
    assert c.h.flags(0).tolist() == [0]
    for _ in range(5):
        c.h.spmv(x, mode=CHECK)
    assert c.h.flags(0).size == 0


def test_spmv_host_entry(O, torch_cuda):
    from paper_conf_dsn_schollbkw16_b200 import AUTOCORRECT, CHECK
    A = MATRICES["st27_11"]()
    c = Case(O, torch_cuda, A)
    x = G.uniform_vector(A.n, 4)
    y = np.empty(A.n)
    nf = c.h.spmv_host(x, y, CHECK | AUTOCORRECT)
    assert nf == 0
    assert_bits_equal(y, O.spmv(A, x), "y via host entry")


def test_nocheck_baseline(O, torch_cuda):
    from paper_conf_dsn_schollbkw16_b200 import NOCHECK
    A = MATRICES["rmat11"]()
    c = Case(O, torch_cuda, A)
    x = G.uniform_vector(A.n, 4)
    y = c.h.spmv(torch_cuda.from_numpy(x).cuda(), mode=NOCHECK)
    assert_bits_equal(y.cpu().numpy(), O.spmv(A, x), "plain y")


# --------------------------------------------------------------------------
# Full size: BASELINE configs[1] (3-D 7-pt 128^3), the bench workload, in the
# launch configuration bench.py times.
# --------------------------------------------------------------------------
def test_full_size_config1(O, torch_cuda):
    A = G.laplacian_3d_7pt(128)
    c = Case(O, torch_cuda, A)
    c.check_encoding()
    ref = c.run(G.uniform_vector(A.n, 42))
    assert ref.flagged.size == 0
    rng = np.random.default_rng(0)
    idx = rng.choice(A.n, 64, replace=False)
    plan = G.FaultPlan(np.zeros(64), np.zeros(64), idx,
                       [G.burst_mask(int(s), 4) for s in rng.integers(0, 64, 64)])
    c.run(G.uniform_vector(A.n, 43), plan=plan)
    c.run(G.uniform_vector(A.n, 44), rate=dict(seed=1, lam=1e-5, targets=0b111, call=3))


# --------------------------------------------------------------------------
# PCG
# --------------------------------------------------------------------------
def _pcg_case(O, torch, A, inj_kw=None, check=True, max_iter=0, literal=False, bscale=1.0):
    from paper_conf_dsn_schollbkw16_b200 import encode
    enc = O.encode(A, 32)
    xs = G.uniform_vector(A.n, 43)
    b = bscale * O.spmv(A, xs)
    x0 = G.uniform_vector(A.n, 44)
    oinj = O.Inject.rate(**inj_kw) if inj_kw else None
    ref = O.pcg(A, enc, b, x0, tol=1e-6, inj=oinj, check=check, max_iter=max_iter,
                literal_stop=literal)
    h = encode(A, 32)
    bd = torch.from_numpy(b).cuda()
    xd = torch.from_numpy(x0.copy()).cuda()
    mi = max_iter if max_iter > 0 else 10 * A.n
    hist = torch.zeros(mi + 1, dtype=torch.float64, device="cuda")
    status, st = h.pcg(bd, xd, tol=1e-6, inject=gpu_inject(rate=inj_kw) if inj_kw else None,
                       check=check, res_hist=hist, max_iter=max_iter, literal_stop=literal)
    torch.cuda.synchronize()
    return ref, status, st, xd.cpu().numpy(), hist.cpu().numpy()[: st["iters"] + 1]


@pytest.mark.parametrize("inj", [None, dict(seed=3, lam=1e-4, targets=0b111)])
def test_pcg_parity(O, torch_cuda, inj):
    A = G.laplacian_3d_7pt(16)
    ref, status, st, x, hist = _pcg_case(O, torch_cuda, A, inj)
    assert status == ref.status == 0
    assert st["iters"] == ref.iters and st["spmv_calls"] == ref.spmv_calls
    assert st["flagged_blocks"] == ref.flagged_blocks
    assert st["recomputed_blocks"] == ref.recomputed_blocks
    assert st["uncorrected_calls"] == ref.uncorrected_calls
    assert np.max(np.abs(hist - ref.res_hist) / np.abs(ref.res_hist)) <= 1e-10
    assert_bits_equal(hist, ref.res_hist, "residual history")
    assert_bits_equal(x, ref.x, "solution")
    if inj:
        assert st["flagged_blocks"] > 0


@pytest.mark.parametrize("inj", [None, dict(seed=4, lam=1e-4, targets=0b111)])
def test_pcg_literal_stop(O, torch_cuda, inj):
    # P:296 read literally (r^T r < eps): bit-exact against the oracle's
    # literal rule, and a different stopping iteration than the relative one
    A = G.laplacian_3d_7pt(16)
    ref, status, st, x, hist = _pcg_case(O, torch_cuda, A, inj, literal=True, bscale=40.0)
    rel, *_ = _pcg_case(O, torch_cuda, A, inj, bscale=40.0)
    assert status == ref.status == 0 and st["iters"] == ref.iters != rel.iters
    assert st["flagged_blocks"] == ref.flagged_blocks
    assert_bits_equal(hist, ref.res_hist, "literal-stop residual history")
    assert_bits_equal(x, ref.x, "literal-stop solution")


def test_pcg_odd_n(O, torch_cuda):
    # odd N: the scratch vectors keep a 16-byte aligned stride (n rounded up)
    A = G.laplacian_3d_7pt(21)  # 9261 rows
    for inj in (None, dict(seed=5, lam=1e-4, targets=0b111)):
        ref, status, st, x, hist = _pcg_case(O, torch_cuda, A, inj)
        assert status == ref.status == 0 and st["iters"] == ref.iters
        assert_bits_equal(hist, ref.res_hist, "odd-n residual history")
        assert_bits_equal(x, ref.x, "odd-n solution")


def test_pcg_unprotected_and_maxiter(O, torch_cuda):
    A = G.laplacian_3d_7pt(12)
    ref, status, st, x, hist = _pcg_case(O, torch_cuda, A, dict(seed=3, lam=1e-5), check=False)
    assert status == ref.status and st["iters"] == ref.iters
    assert_bits_equal(hist, ref.res_hist, "unprotected history")
    ref, status, st, x, hist = _pcg_case(O, torch_cuda, A, None, max_iter=7)
    assert status == ref.status == -5 and st["iters"] == ref.iters == 7
    assert_bits_equal(hist, ref.res_hist, "truncated history")
    assert_bits_equal(x, ref.x, "truncated solution")


def test_irregular_path_routing(O, torch_cuda):
    # power-law rows take k_irr; a lean majority
    # keeps k_lean and sends only the long-row groups to k_irr; hub rows stay
    # with k_general
    from paper_conf_dsn_schollbkw16_b200 import encode
    info = encode(MATRICES["rmat11"]()).info()
    assert info["irr_groups"] > 0 and info["lean"] == 0, info
    info = encode(MATRICES["mixed_lean_irr"]()).info()
    assert info["lean"] == 1 and info["irr_groups"] >= 3 and info["general_groups"] >= 2, info
    info = encode(MATRICES["hubs"]()).info()
    assert info["irr_groups"] > 0 and info["general_groups"] > 0, info


@pytest.mark.parametrize("c_csr", [False, True])
@pytest.mark.parametrize("name", ["rmat11", "mixed_lean_irr", "hubs"])
def test_irregular_faults(O, torch_cuda, name, c_csr):
    # list faults into y rows, t1 and t2 of irregular groups (k_irr's INJECT
    # instantiation), then a rate-mode call at b_s = 32
    A = MATRICES[name]()
    c = Case(O, torch_cuda, A, c_csr=c_csr)
    rl = np.diff(A.row_ptr)
    long_rows = np.nonzero(rl > 32)[0][:3]
    blocks = sorted({int(r) // 32 for r in long_rows})
    plan = G.FaultPlan([0] * (len(long_rows) + 2 * len(blocks)),
                       [0] * len(long_rows) + [1] * len(blocks) + [2] * len(blocks),
                       [int(r) for r in long_rows] + blocks + blocks,
                       [1 << 62] * len(long_rows) + [1 << 61] * len(blocks) + [1 << 60] * len(blocks))
    ref = c.run(G.uniform_vector(A.n, 21), plan=plan)
    assert set(blocks) <= set(ref.flagged.tolist())
    c.run(G.uniform_vector(A.n, 22), rate=dict(seed=9, lam=1e-4, targets=0b111, call=3))


@pytest.mark.parametrize("bs", [64, 128, 512])
@pytest.mark.parametrize("name", ["lap3d_ragged", "rmat11", "hubs", "lap2d_64"])
def test_big_block_sizes(O, torch_cuda, name, bs):
    # b_s beyond a warp (kernels_bigblock.cuh) -- C, K, y, t1,
    # t2, flags and corrections bit-exact against the oracle
    A = MATRICES[name]()
    c = Case(O, torch_cuda, A, bs=bs)
    c.check_encoding()
    ref = c.run(G.uniform_vector(A.n, 7))
    assert ref.flagged.size == 0
    nb = c.enc.nb
    plan = G.FaultPlan([0, 0, 0, 1], [0, 1, 2, 0], [A.n // 2, 0, nb - 1, A.n // 2],
                       [1 << 62, 1 << 61, 1 << 60, 1 << 59])
    ref = c.run(G.uniform_vector(A.n, 8), plan=plan)
    assert ref.flagged.size >= 1
    c.run(G.uniform_vector(A.n, 9), rate=dict(seed=2, lam=1e-4, targets=0b111, call=1))


def test_host_pipelined_matches_device(O, torch_cuda):
    # abft_spmv_host_pipelined (include/abft.h): per-step host x in, y out,
    # copies overlapped across steps -- same bits as the device call and the
    # oracle, per step
    from paper_conf_dsn_schollbkw16_b200 import AUTOCORRECT, CHECK, encode
    A = MATRICES["lap3d_ragged"]()
    h = encode(A, 32)
    torch = torch_cuda
    xs = [torch.from_numpy(G.uniform_vector(A.n, 60 + k)).pin_memory() for k in range(5)]
    ys = [torch.empty(A.n, dtype=torch.float64).pin_memory() for _ in range(5)]
    nf = h.spmv_host_pipelined([x.numpy() for x in xs], [y.numpy() for y in ys],
                               CHECK | AUTOCORRECT)
    assert nf.tolist() == [0] * 5
    for k in range(5):
        assert_bits_equal(ys[k].numpy(), O.spmv(A, xs[k].numpy()), f"y step {k}")


@pytest.mark.parametrize("name", ["st27_11", "lap3d_ragged", "mixed_lean_irr", "rand_empty"])
def test_lean_columns_from_global(O, torch_cuda, name, monkeypatch):
    # COLG: k_lean reading A's columns from global memory
    # instead of staging them -- same bits, error-free and with faults
    monkeypatch.setenv("ABFT_COLG", "1")
    monkeypatch.setenv("ABFT_FORCE_COLG", "1")
    monkeypatch.setenv("ABFT_NO_POS", "1")  # k_lean streams the slot-map records
    A = MATRICES[name]()
    c = Case(O, torch_cuda, A)
    monkeypatch.delenv("ABFT_FORCE_COLG")
    monkeypatch.delenv("ABFT_COLG")
    monkeypatch.delenv("ABFT_NO_POS")
    c.check_encoding()
    ref = c.run(G.uniform_vector(A.n, 31))
    assert ref.flagged.size == 0
    plan = G.FaultPlan([0, 0], [0, 1], [A.n // 3, 0], [1 << 62, 1 << 61])
    c.run(G.uniform_vector(A.n, 32), plan=plan)


def test_lean_runs_large(O, torch_cuda, monkeypatch):
    # LeanRuns (kernels_spmv.cuh): more groups than one 16-group run per warp
    # -> interleaved runs (forced: x of 160^3 fits L2); bit-exact y / t1 /
    # t2 / flags error-free, and with faults (the INJECT kernels walk
    # contiguous ranges) corrections
    monkeypatch.setenv("ABFT_FORCE_RUNS", "1")
    monkeypatch.setenv("ABFT_NO_POS", "1")
    A = G.laplacian_3d_7pt(160)
    c = Case(O, torch_cuda, A)
    monkeypatch.delenv("ABFT_FORCE_RUNS")
    monkeypatch.delenv("ABFT_NO_POS")
    info = c.h.info()
    assert info["lean_runs"] == 1 and info["lean_short"] == 1, info
    ref = c.run(G.uniform_vector(A.n, 34))
    assert ref.flagged.size == 0
    plan = G.FaultPlan([0, 0, 0], [0, 1, 2], [A.n - 5, 4000, 12345], [1 << 62, 1 << 61, 1 << 60])
    ref = c.run(G.uniform_vector(A.n, 33), plan=plan)
    assert ref.flagged.size == 3


def test_config0_single_fault_sweep(O, torch_cuda):
    # BASELINE configs[0] / SURVEY §8(d) config 1: one seeded burst per run on
    # a uniformly chosen y element, 1000 runs: round-0 flags,
    # pre-correction y and corrected y bit-exact against the oracle, run by run
    from paper_conf_dsn_schollbkw16_b200 import AUTOCORRECT, CHECK, Inject, encode
    torch = torch_cuda
    A = G.laplacian_2d_5pt(64)
    enc = O.encode(A, 32)
    h = encode(A, 32)
    xh = G.uniform_vector(A.n, 42)
    x = torch.from_numpy(xh).cuda()
    y0 = O.spmv(A, xh)
    flagged_runs = 0
    for seed in range(1000):
        plan = G.single_fault_plan(A.n, seed)
        ref = O.abft_spmv(A, enc, xh, O.Inject.from_plan(plan), 4)
        y = h.spmv(x, inject=Inject.from_plan(plan), mode=CHECK | AUTOCORRECT)
        fl = h.flags(0)
        assert np.array_equal(fl, ref.flags[0]), (seed, fl, ref.flags[0])
        yc = y.cpu().numpy()
        assert_bits_equal(yc, ref.y, f"corrected y, seed {seed}")
        if fl.size:
            flagged_runs += 1
            assert_bits_equal(yc, y0, f"corrected y == fault-free y, seed {seed}")
    assert flagged_runs > 500


@pytest.mark.parametrize("name", ["7pt128", "27pt128", "rmat20", "7pt192"])
def test_bench_workloads_full_size(O, torch_cuda, name):
    # the bench's own workloads at full size, in the launch configuration
    # bench.py times (7-pt 128^3 = configs[1]: k_lean SHORT; 27-pt 128^3: the
    # general k_lean; R-MAT scale 20: k_irr + k_hub + k_general), every output
    # against the oracle with faults in y, t1 and t2
    # (7-pt 192^3, the PCG matrix: x > 40 MB, so the deferred-butterfly
    # instantiation runs)
    A = {"7pt128": lambda: G.laplacian_3d_7pt(128), "27pt128": lambda: G.stencil_3d_27pt(128),
         "rmat20": lambda: G.rmat(20, 16, 1), "7pt192": lambda: G.laplacian_3d_7pt(192)}[name]()
    c = Case(O, torch_cuda, A)
    ref = c.run(G.uniform_vector(A.n, 42))
    assert ref.flagged.size == 0
    nb = c.enc.nb
    plan = G.FaultPlan([0, 0, 0, 0], [0, 0, 1, 2], [7, A.n - 1, nb // 2, nb - 3],
                       [1 << 62, 1 << 55, 1 << 61, 1 << 60])
    ref = c.run(G.uniform_vector(A.n, 43), plan=plan)
    assert ref.flagged.size >= 3


def test_compact_c_with_huge_hub_row(O, torch_cuda):
    # a block whose A segment exceeds the uint16 slot range keeps an unmapped
    # compact record (k_general streams CSR C for it); every other block is
    # compact -- parity with faults, including in the huge block
    from paper_conf_dsn_schollbkw16_b200 import encode
    rng = np.random.Generator(np.random.PCG64(23))
    n = 80000
    lens = rng.integers(1, 9, n)
    lens[40001] = 70000
    cols = [np.sort(rng.choice(n, size=int(L), replace=False)) for L in lens]
    rp = np.zeros(n + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    col = np.concatenate(cols).astype(np.int32)
    A = G.CSR(rp.astype(np.int32), col, rng.uniform(-1, 1, col.size), "huge_hub")
    info = encode(A).info()
    assert info["c_format_name"] != "csr-f64", info
    c = Case(O, torch_cuda, A)
    assert c.run(G.uniform_vector(n, 3)).flagged.size == 0
    plan = G.FaultPlan([0, 0, 0], [0, 0, 1], [40001, 17, 40001 // 32], [1 << 62, 1 << 61, 1 << 60])
    ref = c.run(G.uniform_vector(n, 4), plan=plan)
    assert set([40001 // 32, 0]) <= set(ref.flagged.tolist())


@pytest.mark.parametrize("lam", [1e-5, 1e-3])
def test_resident_plan(O, torch_cuda, lam):
    # ABFT_INJ_RESIDENT: the plan abft_inject_prepare builds is exactly the
    # oracle's rate plan of that call (R13), and protected calls reusing it
    # repeat the rate-mode call bit for bit (same faults, no plan generation).
    from paper_conf_dsn_schollbkw16_b200 import AUTOCORRECT, CHECK, Inject, encode
    A = MATRICES["lap3d_16"]()
    enc = O.encode(A, 32)
    h = encode(A)
    x = G.uniform_vector(A.n, 21)
    spec = dict(seed=31, lam=lam, targets=0b111, call=2)
    ref = O.abft_spmv(A, enc, x, O.Inject.rate(**spec))
    h.inject_prepare(Inject.rate(**spec), CHECK | AUTOCORRECT)
    ro, ta, ix, mk = h.inject_list()
    oro, ota, oix, omk = O.rate_plan(A, enc, O.Inject.rate(**spec))
    def combined(*cols):  # equal (round, target, index) entries XOR together
        comb = {}
        for r, t, i, m in zip(*cols):
            comb[(int(r), int(t), int(i))] = comb.get((int(r), int(t), int(i)), 0) ^ int(m)
        return sorted(comb.items())
    exp = combined(oro, ota, oix, omk)
    assert combined(ro, ta, ix, mk) == exp and len(exp) > 0
    assert np.all(np.diff(ro.astype(np.int64) * 4 + ta) >= 0)  # keys ascending
    xd = torch_cuda.from_numpy(x).cuda()
    for _ in range(2):
        y = h.spmv(xd, inject=Inject.resident(), mode=CHECK | AUTOCORRECT)
        torch_cuda.cuda.synchronize()
        assert_bits_equal(y.cpu().numpy(), ref.y, "y (resident plan)")
        for r in range(5):
            assert np.array_equal(h.flags(r), ref.flags[r]), r
    # harness control: same lookups, zeroed masks -> the fault-free result
    h.inject_clear_masks()
    y = h.spmv(xd, inject=Inject.resident(), mode=CHECK | AUTOCORRECT)
    torch_cuda.cuda.synchronize()
    assert_bits_equal(y.cpu().numpy(), O.spmv(A, x), "y (cleared masks)")
    assert h.flags(0).size == 0


@pytest.mark.parametrize("c_csr", [False, True])
@pytest.mark.parametrize("name", ["rmat11", "rmat11_natural", "hubs", "rand_empty", "rand_dense"])
def test_popularity_ordered_x(O, torch_cuda, name, c_csr, monkeypatch):
    # the irregular path gathers x through a copy ordered by
    # column popularity (renumbered column arrays, one scatter of x per call)
    # -- only where x_j is read from changes, so y, t1, t2, beta, the flags of
    # every round and the corrected y stay bit-exact against the oracle
    from paper_conf_dsn_schollbkw16_b200 import encode
    monkeypatch.setenv("ABFT_COLPERM", "1")
    A = MATRICES[name]()
    info = encode(A, c_csr=c_csr).info()
    if info["lean"] or info["stream"]:
        pytest.skip("staged / position-map path: no reordering")
    assert info["col_perm"] == 1, info
    c = Case(O, torch_cuda, A, c_csr=c_csr)
    assert c.h.info()["col_perm"] == 1
    assert c.run(G.uniform_vector(A.n, 31)).flagged.size == 0
    rl = np.diff(A.row_ptr)
    rows = np.nonzero(rl > 0)[0]
    r0, r1 = int(rows[0]), int(rows[-1])
    plan = G.FaultPlan([0, 0, 0, 1], [0, 0, 1, 0], [r0, r1, r1 // 32, r1],
                       [1 << 62, 1 << 58, 1 << 61, 1 << 62])
    ref = c.run(G.uniform_vector(A.n, 32), plan=plan)
    assert {r0 // 32, r1 // 32} <= set(ref.flagged.tolist())
    c.run(G.uniform_vector(A.n, 33), rate=dict(seed=5, lam=1e-3, targets=0b111, call=1))
    monkeypatch.setenv("ABFT_COLPERM", "0")
    assert encode(A, c_csr=c_csr).info()["col_perm"] == 0


def test_popularity_ordered_x_unaligned_operand(O, torch_cuda, monkeypatch):
    # k_xperm's scalar path (x not 16-B aligned: a view one element into a
    # buffer) gives the same bits as the oracle
    from paper_conf_dsn_schollbkw16_b200 import CHECK, encode
    monkeypatch.setenv("ABFT_COLPERM", "1")
    torch = torch_cuda
    A = MATRICES["rmat11"]()
    h = encode(A)
    assert h.info()["col_perm"] == 1
    x = G.uniform_vector(A.n, 61)
    enc = O.encode(A, 32)
    ref = O.abft_spmv(A, enc, x, None, 4)
    buf = torch.zeros(A.n + 1, dtype=torch.float64, device="cuda")
    buf[1:] = torch.from_numpy(x).cuda()
    xv = buf[1:]
    assert xv.data_ptr() % 16 != 0
    y = h.spmv(xv, mode=CHECK)
    torch.cuda.synchronize()
    assert_bits_equal(y.cpu().numpy(), ref.y_pre, "y")
    assert np.array_equal(h.flags(0), ref.flags[0])


@pytest.mark.parametrize("name", ["27pt256", "rmat24"])
def test_full_size_properties(torch_cuda, name):
    # configs[3] / configs[2] at full size in the bench's launch configuration
    # (too large for the oracle within seconds): properties that hold at any
    # size -- no flag on a fault-free call (the bound); every injected
    # fault far above tau flagged and localized to its own block (y rows)
    # or its block (t1 / t2); the correction restores the fault-free y bit
    # for bit; the unprotected kernel computes the same y.
    from paper_conf_dsn_schollbkw16_b200 import CHECK, Inject, encode
    torch = torch_cuda
    A = {"27pt256": lambda: G.stencil_3d_27pt(256), "rmat24": lambda: G.rmat(24, 16, 1)}[name]()
    h = encode(A, 32)
    x = torch.from_numpy(G.uniform_vector(A.n, 42)).cuda()
    y0 = h.spmv(x, mode=CHECK)
    torch.cuda.synchronize()
    assert h.flags(0).size == 0
    yp = h.spmv(x, mode=0)
    torch.cuda.synchronize()
    assert torch.equal(yp.view(torch.int64), y0.view(torch.int64))
    nb = (A.n + 31) // 32
    rows = [5, A.n // 3, A.n - 1]
    blocks = [nb // 2 + 1, nb - 2]
    plan = G.FaultPlan([0] * 5, [0, 0, 0, 1, 2], rows + blocks,
                       [1 << 62, 1 << 62, 1 << 62, 1 << 62, 1 << 62])
    y = h.spmv(x, inject=Inject.from_plan(plan), mode=CHECK)
    torch.cuda.synchronize()
    want = sorted({r // 32 for r in rows} | set(blocks))
    assert sorted(h.flags(0).tolist()) == want
    h.correct(x, y, 4, inject=Inject.from_plan(plan))
    torch.cuda.synchronize()
    assert h.flags(1).size == 0
    assert torch.equal(y.view(torch.int64), y0.view(torch.int64))
