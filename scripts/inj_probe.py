"""Kernel list of protected calls: fault-free vs a resident (empty) plan."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_dsn_schollbkw16_b200 import AUTOCORRECT, CHECK, Inject, encode
from paper_conf_dsn_schollbkw16_b200 import inputs as G
A = G.laplacian_3d_7pt(128)
h = encode(A)
x = torch.from_numpy(G.uniform_vector(A.n, 42)).cuda()
y = torch.empty_like(x)
m = CHECK | AUTOCORRECT
lam = float(sys.argv[1]) if len(sys.argv) > 1 else 1e-8
for _ in range(3):
    h.spmv(x, y, mode=m)
h.inject_prepare(Inject.rate(seed=77, lam=lam, call=0), m)
torch.cuda.synchronize()
for _ in range(3):
    h.spmv(x, y, inject=Inject.resident(), mode=m)
torch.cuda.synchronize()
