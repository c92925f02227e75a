"""One protected PCG solve on 192^3 (for an ncu launch list)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_dsn_schollbkw16_b200 import Inject, encode, inputs as G
n3 = int(sys.argv[1]) if len(sys.argv) > 1 else 192
check = (sys.argv[2] != "0") if len(sys.argv) > 2 else True
lam = float(sys.argv[3]) if len(sys.argv) > 3 else 0.0
A = G.laplacian_3d_7pt(n3)
h = encode(A, 32)
xs = torch.from_numpy(G.uniform_vector(A.n, 43)).cuda()
b = h.spmv(xs, mode=0)
x = torch.from_numpy(G.uniform_vector(A.n, 44)).cuda()
st, stats = h.pcg(b, x, tol=1e-6, check=check, max_iter=20,
                  inject=Inject.rate(seed=7, lam=lam) if lam > 0 else None)
torch.cuda.synchronize()
print(st, stats)
