"""GPU parity of the related-work baseline: dense check
[30, 31] + complete recomputation [31] through the C ABI against the oracle
(oracle/abft_oracle.c or_dense_*): c, K35, t1, t2, beta, tau and the per-round
flags bit-exact, y bit-exact before and after recomputation."""
import numpy as np
import pytest

from paper_conf_dsn_schollbkw16_b200 import inputs as G

from test_gpu_parity import MATRICES, assert_bits_equal, gpu_inject, oracle_inject

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    return torch


def scale_mask(v, f=2.0 ** 20):
    return int(np.float64(v * f).view(np.uint64) ^ np.float64(v).view(np.uint64))


def run_pair(O, torch, A, x, plan=None, bound35=False, correct=True, max_rounds=4):
    from paper_conf_dsn_schollbkw16_b200 import encode
    h = encode(A, 32, max_rounds).dense_encode()
    e = O.dense_encode(A)
    assert_bits_equal(h.dense_checksum(), e.c, "c")
    ref = O.dense_spmv(A, e, x, bound35=bound35, inj=oracle_inject(O, plan),
                       max_rounds=max_rounds if correct else 0)
    xd = torch.from_numpy(x).cuda()
    y = h.spmv_dense(xd, inject=gpu_inject(plan), correct=correct, bound35=bound35)
    torch.cuda.synchronize()
    r = h.dense_result()
    assert r["k35"] == e.k35
    assert_bits_equal([r["t1"], r["t2"], r["beta"], r["tau"]], [ref.t1, ref.t2, ref.beta, ref.tau],
                      "t1 t2 beta tau")
    n = (max_rounds if correct else 0) + 1
    assert r["flag_rounds"][:n].tolist() == ref.flag_rounds.tolist()
    assert_bits_equal(y.cpu().numpy(), ref.y, "y")
    return ref, r


@pytest.mark.parametrize("name", ["lap2d_64", "lap3d_ragged", "st27_11", "rand_empty", "rmat11",
                                  "hubs", "mixed_lean_irr", "tiny1", "all_empty"])
@pytest.mark.parametrize("bound35", [False, True])
def test_dense_error_free(torch_cuda, O, name, bound35):
    A = MATRICES[name]()
    ref, _ = run_pair(O, torch_cuda, A, G.uniform_vector(A.n, 11), bound35=bound35)
    assert ref.flag_rounds.sum() == 0


@pytest.mark.parametrize("name", ["lap3d_16", "rmat11", "mixed_lean_irr"])
def test_dense_fault_recompute(torch_cuda, O, name):
    A = MATRICES[name]()
    x = G.uniform_vector(A.n, 12)
    y = O.spmv(A, x)
    i = int(np.argmax(np.abs(y)))
    plan = G.FaultPlan([0], [0], [i], [scale_mask(y[i])])
    ref, r = run_pair(O, torch_cuda, A, x, plan=plan)
    assert ref.flag_rounds[0] == 1 and ref.flag_rounds[1:].sum() == 0


def test_dense_faults_every_round(torch_cuda, O):
    A = MATRICES["lap3d_16"]()
    x = G.uniform_vector(A.n, 13)
    y = O.spmv(A, x)
    e = O.dense_encode(A)
    t1 = O.dense_spmv(A, e, x).t1
    plan = G.FaultPlan([0, 1, 2], [0, 1, 2], [5, 0, 0],
                       [scale_mask(y[5]), scale_mask(t1), scale_mask(t1)])
    ref, _ = run_pair(O, torch_cuda, A, x, plan=plan, max_rounds=2)
    assert ref.status == -6 and ref.flag_rounds.tolist() == [1, 1, 1]


def test_dense_detect_only(torch_cuda, O):
    A = MATRICES["lap2d_64"]()
    x = G.uniform_vector(A.n, 14)
    y = O.spmv(A, x)
    plan = G.FaultPlan([0], [0], [7], [scale_mask(y[7])])
    ref, _ = run_pair(O, torch_cuda, A, x, plan=plan, correct=False)
    assert ref.flag_rounds.tolist() == [1]


# --------------------------------------------------------------------------
# Checkpoint-rollback PCG baseline vs or_pcg_cr
# --------------------------------------------------------------------------
def _cr_case(O, torch, A, inj_kw=None, max_iter=0):
    from paper_conf_dsn_schollbkw16_b200 import encode
    den = O.dense_encode(A)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    oinj = O.Inject.rate(**inj_kw) if inj_kw else None
    ref = O.pcg_cr(A, den, b, x0, tol=1e-6, inj=oinj, max_iter=max_iter)
    h = encode(A, 32).dense_encode()
    bd = torch.from_numpy(b).cuda()
    xd = torch.from_numpy(x0.copy()).cuda()
    mi = max_iter if max_iter > 0 else 10 * A.n
    hist = torch.zeros(mi + 1, dtype=torch.float64, device="cuda")
    status, st = h.pcg(bd, xd, tol=1e-6, inject=gpu_inject(rate=inj_kw) if inj_kw else None,
                       check="checkpoint", res_hist=hist, max_iter=max_iter)
    torch.cuda.synchronize()
    return ref, status, st, xd.cpu().numpy(), hist.cpu().numpy()[: st["iters"] + 1]


@pytest.mark.parametrize("inj", [None, dict(seed=9, lam=1e-4, targets=1),
                                 dict(seed=5, lam=3e-4, targets=1, call=11)])
def test_pcg_checkpoint_parity(O, torch_cuda, inj):
    A = G.laplacian_3d_7pt(8) if inj else G.laplacian_3d_7pt(16)
    ref, status, st, x, hist = _cr_case(O, torch_cuda, A, inj)
    assert status == ref.status
    assert st["iters"] == ref.iters and st["spmv_calls"] == ref.spmv_calls
    assert st["flagged_blocks"] == ref.rollbacks
    assert st["recomputed_blocks"] == ref.executed - ref.iters - ref.rollbacks
    assert_bits_equal(hist, ref.res_hist, "residual history")
    assert_bits_equal(x, ref.x, "solution")
    if inj and inj["seed"] == 9:
        assert ref.rollbacks > 0


def test_dense_rate_mode(O, torch_cuda):
    # rate faults on the dense-check SpMV: the y-only plan (R25), both sides
    A = MATRICES["lap3d_16"]()
    x = G.uniform_vector(A.n, 15)
    from paper_conf_dsn_schollbkw16_b200 import encode
    h = encode(A, 32).dense_encode()
    e = O.dense_encode(A)
    rate = dict(seed=4, lam=1e-4, targets=1, call=2)
    ref = O.dense_spmv(A, e, x, inj=O.Inject.rate(**rate))
    y = h.spmv_dense(torch_cuda.from_numpy(x).cuda(), inject=gpu_inject(rate=rate))
    r = h.dense_result()
    assert r["flag_rounds"].tolist() == ref.flag_rounds.tolist()
    assert_bits_equal([r["t1"], r["t2"]], [ref.t1, ref.t2], "t1 t2")
    assert_bits_equal(y.cpu().numpy(), ref.y, "y")
