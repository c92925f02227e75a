"""PCG time-to-solution on 192^3, protected and unprotected, CUDA events
(A/B of builds via ABFT_LIB; the bench's --pcg also runs the baselines)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_dsn_schollbkw16_b200 import encode, inputs as G
n3 = int(sys.argv[1]) if len(sys.argv) > 1 else 192
A = G.laplacian_3d_7pt(n3)
h = encode(A, 32)
xs = torch.from_numpy(G.uniform_vector(A.n, 43)).cuda()
b = h.spmv(xs, mode=0)
x0 = torch.from_numpy(G.uniform_vector(A.n, 44)).cuda()
out = {}
for check in (False, True):
    ts = []
    for rep in range(4):
        x = x0.clone()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        st, stats = h.pcg(b, x, tol=1e-6, check=check)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    out["protected" if check else "unprotected"] = (round(min(ts[1:]), 3), stats["iters"])
print(os.environ.get("ABFT_LIB", "default").split("/")[-1], out)
