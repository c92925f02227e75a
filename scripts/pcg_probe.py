"""One protected PCG solve at 192^3 with rate faults (targets from argv)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_dsn_schollbkw16_b200 import Inject, encode
from paper_conf_dsn_schollbkw16_b200 import inputs as G
lam, targets = float(sys.argv[1]), int(sys.argv[2])
n3 = int(sys.argv[3]) if len(sys.argv) > 3 else 192
A = G.laplacian_3d_7pt(n3)
h = encode(A, 32, 4)
b = h.spmv(torch.from_numpy(G.uniform_vector(A.n, 43)).cuda(), mode=0)
x0 = torch.from_numpy(G.uniform_vector(A.n, 44)).cuda()
for rep in range(2):
    x = x0.clone()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    st, s = h.pcg(b, x, tol=1e-6, inject=Inject.rate(seed=7, lam=lam, targets=targets) if lam > 0 else None)
    torch.cuda.synchronize()
    print(rep, st, s, time.perf_counter() - t0, flush=True)
