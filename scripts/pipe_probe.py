"""Probe abft_spmv_host_pipelined overlap: default (legacy) stream vs an
explicit non-blocking stream, NOCHECK vs CHECK."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_dsn_schollbkw16_b200 import encode, inputs as G, CHECK, AUTOCORRECT, NOCHECK
A = G.laplacian_3d_7pt(128)
h = encode(A)
xp = torch.from_numpy(G.uniform_vector(A.n, 42)).pin_memory()
yp = torch.empty(A.n, dtype=torch.float64).pin_memory()
xn, yn = xp.numpy(), yp.numpy()
from paper_conf_dsn_schollbkw16_b200.abft import PinnedArray
px, py = PinnedArray(A.n), PinnedArray(A.n)
px.a[:] = xn
ns = torch.cuda.Stream()
for label, st, mode in [("legacy CHECK", None, CHECK | AUTOCORRECT), ("nonblocking CHECK", ns, CHECK | AUTOCORRECT),
                        ("legacy NOCHECK", None, NOCHECK), ("lib-pinned CHECK", None, CHECK | AUTOCORRECT)]:
    if label.startswith("lib"):
        xn, yn = px.a, py.a
    h.spmv_host_pipelined([xn] * 4, [yn] * 4, mode, stream=st)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h.spmv_host_pipelined([xn] * 100, [yn] * 100, mode, stream=st)
    print(label, (time.perf_counter() - t0) / 100 * 1e3, "ms/step")
