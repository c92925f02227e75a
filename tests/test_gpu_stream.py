"""GPU parity of the warp-specialized fused kernel (k_stream) and its
position-map checksum records against the CPU oracle:
y, t1, t2, beta, the flags of every round and the corrected y bit for bit,
error-free and with faults in y / t1 / t2, in list and rate mode, over
row-regular matrices (the format's home: stencils with boundary exception
rows) and forced onto irregular ones (every row an exception, empty rows,
long rows on the general path), several value types, chunk sizes and ring
depths."""
import numpy as np
import pytest

from paper_conf_dsn_schollbkw16_b200 import inputs as G
from test_gpu_parity import Case, assert_bits_equal

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    from paper_conf_dsn_schollbkw16_b200 import _build
    _build.build()
    return torch


def _halves(n, density, seed):
    # values k / 2: exact in float32, not integers -> the f32 record type
    A = G.random_csr(n, density, seed)
    rng = np.random.default_rng(seed)
    return G.CSR(A.row_ptr, A.col, rng.integers(-64, 64, A.col.size) / 2.0, "halves")


def _mixed_long(n=3000, seed=5):
    # mostly short rows; a few rows of 40..300 entries make their groups
    # ineligible (general path) inside otherwise streamed chunks
    rng = np.random.Generator(np.random.PCG64(seed))
    lens = rng.integers(0, 10, n)
    lens[[100, 1500, 2999]] = [40, 300, 64]
    cols = [np.sort(rng.choice(n, size=int(L), replace=False)) for L in lens]
    rp = np.zeros(n + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    col = np.concatenate(cols).astype(np.int32)
    return G.CSR(rp.astype(np.int32), col, rng.uniform(-1, 1, col.size), "mixed_long")


# (matrix, force the format onto it, expected value type)
FAMILIES = {
    "lap2d_64": (lambda: G.laplacian_2d_5pt(64), False, "int8+pos"),
    "lap3d_32": (lambda: G.laplacian_3d_7pt(32), False, "int8+pos"),
    "lap3d_16": (lambda: G.laplacian_3d_7pt(16), False, "int8+pos"),
    "lap3d_40x24x9": (lambda: G.laplacian_3d_7pt(40, 24, 9), True, "int8+pos"),
    "st27_32": (lambda: G.stencil_3d_27pt(32, 12, 6), False, "int8+pos"),
    "st27_11": (lambda: G.stencil_3d_27pt(11), True, "int8+pos"),
    "rand_f64": (lambda: G.random_csr(2048, 0.004, 3), True, "f64+pos"),
    "rand_empty": (lambda: G.random_csr(1500, 0.003, 4, empty_rows=0.3), True, "f64+pos"),
    "rand_int16": (lambda: G.random_csr(1024, 0.01, 6, integer=True, max_int=300), True,
                   "int16+pos"),
    "halves_f32": (lambda: _halves(1024, 0.01, 7), True, "f32+pos"),
    "mixed_long": (lambda: _mixed_long(), True, "f64+pos"),
}


def make_case(O, torch, name, monkeypatch, **env):
    mk, force, fmt = FAMILIES[name]
    A = mk()
    if force:
        monkeypatch.setenv("ABFT_FORCE_POS", "1")
    for k, v in env.items():
        monkeypatch.setenv(k, str(v))
    c = Case(O, torch, A)
    for k in list(env) + (["ABFT_FORCE_POS"] if force else []):
        monkeypatch.delenv(k)
    info = c.h.info()
    assert info["c_format_name"] == fmt, info
    assert info["stream"] == 1, info
    return A, c


@pytest.mark.parametrize("name", sorted(FAMILIES))
def test_stream_parity(O, torch_cuda, name, monkeypatch):
    A, c = make_case(O, torch_cuda, name, monkeypatch)
    c.check_encoding()
    ref = c.run(G.uniform_vector(A.n, 42))
    assert ref.flagged.size == 0
    nb = c.enc.nb
    rng = np.random.default_rng(len(name))
    idx = rng.choice(A.n, 6, replace=False)
    plan = G.FaultPlan(np.zeros(9), [0] * 6 + [1, 2, 1], list(idx) + [nb // 2, nb - 1, 0],
                       [1 << 62, 1 << 55, 1 << 40, 1 << 61, 1 << 20, 1 << 63, 1 << 60, 1 << 59,
                        1 << 58])
    ref = c.run(G.uniform_vector(A.n, 43), plan=plan)
    assert ref.flagged.size >= 3
    for call in range(2):
        c.run(G.uniform_vector(A.n, 44 + call), rate=dict(seed=7, lam=1e-3, targets=0b111, call=call))


@pytest.mark.parametrize("G_,NS", [(2, 2), (4, 3), (8, 2), (8, 5)])
@pytest.mark.parametrize("name", ["lap3d_16", "st27_11", "rand_empty"])
def test_stream_chunk_and_ring_shapes(O, torch_cuda, name, G_, NS, monkeypatch):
    # groups per chunk / ring depth change the producer's chunking, the ring
    # wrap-around and the partial last chunk -- never the bits
    if name == "st27_11" and G_ == 8:
        pytest.skip("27-pt chunks of 8 groups exceed the ring budget")
    A, c = make_case(O, torch_cuda, name, monkeypatch, ABFT_STREAM_G=G_, ABFT_STREAM_NS=NS)
    info = c.h.info()
    assert info["stream_g"] == G_ and info["stream_stages"] <= NS, info
    assert c.run(G.uniform_vector(A.n, 12)).flagged.size == 0
    plan = G.FaultPlan([0, 0], [0, 2], [A.n - 1, 1], [1 << 62, 1 << 61])
    c.run(G.uniform_vector(A.n, 13), plan=plan)


@pytest.mark.parametrize("name", ["lap3d_32", "st27_32", "mixed_long"])
def test_stream_plain_kernel(O, torch_cuda, name, monkeypatch):
    # CHECK = false: the same kernel streams row pointers instead of records
    from paper_conf_dsn_schollbkw16_b200 import NOCHECK
    A, c = make_case(O, torch_cuda, name, monkeypatch)
    x = G.uniform_vector(A.n, 4)
    y = c.h.spmv(torch_cuda.from_numpy(x).cuda(), mode=NOCHECK)
    assert_bits_equal(y.cpu().numpy(), O.spmv(A, x), "plain y")


def _exception_rows(O, A):
    # brute force of the record's definition (kernels_stream.cuh): row l of
    # group g has C positions P_l; it is regular iff it is no longer than the
    # typical row (the best of lanes 1, 15, 16, 30) and P_l - l agrees with
    # the typical row's P_c - c on its own entries
    enc = O.encode(A, 32)
    tot = 0
    for g in range(A.n // 32):
        cr = enc.col[enc.row_ptr[g]:enc.row_ptr[g + 1]]
        W = []
        for l in range(32):
            i = 32 * g + l
            cols = A.col[A.row_ptr[i]:A.row_ptr[i + 1]]
            W.append([int(np.searchsorted(cr, c)) - l for c in cols])
        tot += min(sum(1 for l in range(32)
                       if not (len(W[l]) <= len(W[c]) and W[l] == W[c][:len(W[l])]))
                   for c in (1, 15, 16, 30))
    return tot


def test_stream_exception_rows_counted(O, torch_cuda):
    # 7-pt with nx = 128: only x-boundary rows are exceptions (at most one per
    # boundary group, two of every four groups along x), every group streamed
    from paper_conf_dsn_schollbkw16_b200 import encode
    A = G.laplacian_3d_7pt(128, 8, 4)
    info = encode(A).info()
    assert info["c_format_name"] == "int8+pos" and info["stream"] == 1
    assert info["general_groups"] == 0
    exp = _exception_rows(O, A)
    assert 0 < exp <= (A.n // 128) * 2
    assert info["pos_exc_rows"] == exp, (info, exp)


@pytest.mark.parametrize("defer", [0, 1])
def test_stream_pcg_parity(O, torch_cuda, defer, monkeypatch):
    # the PCG case study over the streamed SpMV, with rate faults
    # (immediate and deferred butterflies: the fused p.q rides in it)
    from test_gpu_parity import _pcg_case
    monkeypatch.setenv("ABFT_STREAM_DEFER", str(defer))
    A = G.laplacian_3d_7pt(32)
    for inj in (None, dict(seed=3, lam=1e-5, targets=0b111)):
        ref, status, st, x, hist = _pcg_case(O, torch_cuda, A, inj)
        assert st["iters"] == ref.iters and status == ref.status
        assert_bits_equal(hist, ref.res_hist, "residual history")
        assert_bits_equal(x, ref.x, "x")


@pytest.mark.parametrize("defer", [0, 1])
@pytest.mark.parametrize("name", ["lap3d_32", "lap2d_64", "st27_32", "st27_11", "rand_empty", "rand_int16"])
def test_stream_deferred_butterfly(O, torch_cuda, name, defer, monkeypatch):
    # StreamCfg::defer: a group's reduce-scatter + test runs
    # one consumer step later, after the next group's gathers are issued --
    # the same values, so flags, corrections and the PCG p.q stay bit-exact
    A, c = make_case(O, torch_cuda, name, monkeypatch, ABFT_STREAM_DEFER=defer)
    assert c.run(G.uniform_vector(A.n, 52)).flagged.size == 0
    nb = c.enc.nb
    plan = G.FaultPlan([0, 0, 0, 0], [0, 0, 1, 2], [3, A.n - 1, nb // 3, nb - 1],
                       [1 << 62, 1 << 57, 1 << 61, 1 << 60])
    assert c.run(G.uniform_vector(A.n, 53), plan=plan).flagged.size >= 3
    c.run(G.uniform_vector(A.n, 54), rate=dict(seed=3, lam=1e-3, targets=0b111, call=2))


def _arrow_laplacian(n3=14):
    # SPD: the 7-pt Laplacian plus an "arrow" -- row and column 0 dense with
    # small entries (row 0 has n entries > 1024: a hub row on the general
    # path) -- and a diagonal raised enough to stay diagonally dominant
    L = G.laplacian_3d_7pt(n3)
    n = L.n
    rows = [np.arange(L.row_ptr[i], L.row_ptr[i + 1]) for i in range(n)]
    cols, vals, rp = [], [], [0]
    for i in range(n):
        c = L.col[rows[i]].tolist()
        v = L.val[rows[i]].tolist()
        if i == 0:
            lap = dict(zip(c, v))  # keep the Laplacian's own row-0 entries (symmetric)
            c = list(range(n))
            v = [lap.get(j, 1e-3) for j in range(n)]
            v[0] = 6.0 + 1e-3 * n
        elif 0 not in c:
            c = [0] + c
            v = [1e-3] + v
        cols += c
        vals += v
        rp.append(len(cols))
    return G.CSR(np.array(rp, np.int32), np.array(cols, np.int32), np.array(vals), "arrow")


@pytest.mark.parametrize("inj", [None, dict(seed=5, lam=2e-6, targets=0b111)])
def test_stream_pcg_with_hub_row(O, torch_cuda, inj, monkeypatch):
    # position-map records with one hub row (> 1024 entries, k_hub + k_general)
    # inside a PCG: few candidates per faulty SpMV take k_finish's CTA-0
    # path, which also completes the p.q sum (kernels_pcgfin.cuh)
    from test_gpu_parity import _pcg_case
    from paper_conf_dsn_schollbkw16_b200 import encode
    monkeypatch.setenv("ABFT_FORCE_POS", "1")  # the arrow column makes every row an exception
    A = _arrow_laplacian()
    info = encode(A).info()
    assert info["stream"] == 1 and info["hub_chunks"] > 0, info
    ref, status, st, x, hist = _pcg_case(O, torch_cuda, A, inj)
    assert status == ref.status == 0
    assert st["iters"] == ref.iters and st["flagged_blocks"] == ref.flagged_blocks
    assert_bits_equal(hist, ref.res_hist, "residual history")
    assert_bits_equal(x, ref.x, "x")
    if inj:
        assert ref.flagged_blocks > 0


def test_stream_without_pdl_subprocess(torch_cuda):
    # ABFT_NO_PDL=1 (plain launches instead of programmatic dependent launch;
    # read once per process): the same bits as the oracle
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = (
        "import numpy as np, torch\n"
        "from oracle import oracle as O\n"
        "from paper_conf_dsn_schollbkw16_b200 import CHECK, encode, inputs as G\n"
        "A = G.laplacian_3d_7pt(24)\n"
        "x = G.uniform_vector(A.n, 42)\n"
        "plan = G.FaultPlan([0, 0], [0, 1], [100, 7], [1 << 62, 1 << 61])\n"
        "ref = O.abft_spmv(A, O.encode(A, 32), x, O.Inject.from_plan(plan), 4)\n"
        "from paper_conf_dsn_schollbkw16_b200 import Inject\n"
        "h = encode(A, 32)\n"
        "assert h.info()['stream'] == 1\n"
        "xd = torch.from_numpy(x).cuda()\n"
        "y = h.spmv(xd, inject=Inject.from_plan(plan), mode=CHECK)\n"
        "torch.cuda.synchronize()\n"
        "assert np.array_equal(y.cpu().numpy().view(np.uint64), ref.y_pre.view(np.uint64))\n"
        "assert np.array_equal(h.flags(0), ref.flags[0])\n"
        "h.correct(xd, y, 4, inject=Inject.from_plan(plan))\n"
        "torch.cuda.synchronize()\n"
        "assert np.array_equal(y.cpu().numpy().view(np.uint64), ref.y.view(np.uint64))\n"
        "print('ok')\n")
    env = dict(os.environ, ABFT_NO_PDL="1", PYTHONPATH=root)
    r = subprocess.run([sys.executable, "-c", code], cwd=root, env=env, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr[-2000:]
