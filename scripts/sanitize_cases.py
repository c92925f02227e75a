"""Small runs of every kernel family for compute-sanitizer (memcheck,
racecheck, synccheck, initcheck): k_stream (protected, plain, faults, rate
mode), k_lean (slot-map records), k_irr / k_hub / k_general (R-MAT-like and
hub rows), k_finish with correction rounds (software grid barrier), the dense
check, PCG, the distributed external-exchange path.  Exit code 0 when every
result matches the oracle (the sanitizer's own report is the evidence).

usage: compute-sanitizer --tool memcheck python scripts/sanitize_cases.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    from oracle import oracle as O
    from paper_conf_dsn_schollbkw16_b200 import AUTOCORRECT, CHECK, Dist, Inject, NOCHECK, encode
    from paper_conf_dsn_schollbkw16_b200 import inputs as G
    from paper_conf_dsn_schollbkw16_b200 import parallel as PL
    O.build()
    bad = []

    def spmv_case(name, A, env=None, plan=None, rate=None):
        for k, v in (env or {}).items():
            os.environ[k] = v
        h = encode(A)
        for k in (env or {}):
            del os.environ[k]
        enc = O.encode(A, 32)
        x = G.uniform_vector(A.n, 5)
        oinj = O.Inject.from_plan(plan) if plan is not None else (
            O.Inject.rate(**rate) if rate else None)
        ginj = Inject.from_plan(plan) if plan is not None else (Inject.rate(**rate) if rate else None)
        ref = O.abft_spmv(A, enc, x, oinj)
        xd = torch.from_numpy(x).cuda()
        y = h.spmv(xd, inject=ginj, mode=CHECK | AUTOCORRECT)
        yp = h.spmv(xd, mode=NOCHECK)
        torch.cuda.synchronize()
        ok = np.array_equal(y.cpu().numpy().view(np.uint64), ref.y.view(np.uint64))
        ok = ok and np.array_equal(yp.cpu().numpy().view(np.uint64), O.spmv(A, x).view(np.uint64))
        ok = ok and np.array_equal(h.flags(0), ref.flags[0]) and h.health() == 0
        print(name, h.info()["c_format_name"], "ok" if ok else "MISMATCH", flush=True)
        if not ok:
            bad.append(name)

    lap = G.laplacian_3d_7pt(32, 32, 8)
    plan = G.FaultPlan([0, 0, 0, 1], [0, 1, 2, 0], [77, 40, 90, 77], [1 << 62, 1 << 61, 1 << 60, 1 << 55])
    spmv_case("stream-7pt", lap)
    spmv_case("stream-7pt-faults", lap, plan=plan)
    spmv_case("stream-7pt-rate", lap, rate=dict(seed=3, lam=1e-3, targets=7, call=1))
    spmv_case("stream-27pt", G.stencil_3d_27pt(32, 8, 6), plan=plan)
    spmv_case("lean-7pt", lap, env={"ABFT_NO_POS": "1"}, plan=plan)
    spmv_case("irr-rmat", G.rmat(12, 16, 5), plan=plan)
    spmv_case("hubs", G.hub_csr(5000, 11), plan=plan)
    # correction rounds with many flags: every CTA joins the grid barrier
    many = G.FaultPlan(np.zeros(200), np.zeros(200), np.arange(0, 200 * 40, 40), [1 << 62] * 200)
    spmv_case("finish-grid-rounds", lap, plan=many)
    # dense check + complete recomputation
    A = G.laplacian_3d_7pt(16)
    h = encode(A)
    h.dense_encode()
    x = torch.from_numpy(G.uniform_vector(A.n, 2)).cuda()
    h.spmv_dense(x, inject=Inject.from_plan(G.FaultPlan([0], [0], [5], [1 << 62])))
    torch.cuda.synchronize()
    dr = h.dense_result()
    print("dense", "ok" if dr["flag_rounds"][0] == 1 else f"MISMATCH {dr}", flush=True)
    # PCG (protected, rate faults)
    enc = O.encode(A, 32)
    b = O.spmv(A, G.uniform_vector(A.n, 43))
    x0 = G.uniform_vector(A.n, 44)
    ref = O.pcg(A, enc, b, x0, tol=1e-6, inj=O.Inject.rate(seed=3, lam=1e-4))
    xd = torch.from_numpy(x0.copy()).cuda()
    st, s = h.pcg(torch.from_numpy(b).cuda(), xd, tol=1e-6, inject=Inject.rate(seed=3, lam=1e-4))
    ok = s["iters"] == ref.iters and np.array_equal(xd.cpu().numpy().view(np.uint64),
                                                     ref.x.view(np.uint64))
    print("pcg", "ok" if ok else "MISMATCH", flush=True)
    if not ok:
        bad.append("pcg")
    # distributed, external exchange, 2 logical ranks
    A = G.laplacian_3d_7pt(16, 16, 16)
    ranges = PL.block_partition(A.n, 2)
    rg = PL.ranges_array(ranges)
    dss = [PL.DistSpmv(Dist(r, 2, rg), PL.shard_rows(A, a, b_)) for r, (a, b_) in enumerate(ranges)]
    ex = PL.LocalExchange(dss)
    x = G.uniform_vector(A.n, 9)
    ex.spmv_all({r: torch.from_numpy(x[a:b_].copy()).cuda() for r, (a, b_) in enumerate(ranges)})
    torch.cuda.synchronize()
    y = np.concatenate([d.y.cpu().numpy() for d in dss])
    ok = np.array_equal(y.view(np.uint64), O.spmv(A, x).view(np.uint64))
    print("dist-2", "ok" if ok else "MISMATCH", flush=True)
    if not ok:
        bad.append("dist")
    print("ALL OK" if not bad else f"FAILED: {bad}", flush=True)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
