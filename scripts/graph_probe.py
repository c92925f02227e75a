import time, torch
from paper_conf_dsn_schollbkw16_b200 import inputs as G, parallel as PL
from paper_conf_dsn_schollbkw16_b200.abft import CHECK, DEFER_FINISH, NOCHECK
n3=192
rows = G.stencil_rows("7pt", n3, n3, n3, 0, n3)
sh = PL.make_shard(rows, 0, n3**3, 0, 1, [(0, n3**3)])
d = PL.DistSpmv(sh)
d.own().copy_(torch.from_numpy(G.uniform_vector(sh.n, 43)))
part = torch.empty(1, dtype=torch.float64, device="cuda")
cases = {
 "nocheck": lambda: d.h.spmv(d.x_ext, d.y, mode=NOCHECK),
 "check_defer": lambda: d.h.spmv(d.x_ext, d.y, mode=CHECK | DEFER_FINISH),
 "beta_partial": lambda: d.h.beta_partial(part),
 "torch_add": lambda: d.y.add_(1.0),
}
for name, fn in cases.items():
    for _ in range(3): fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(16): fn()
    e1.record(); torch.cuda.synchronize(); eager = e0.elapsed_time(e1) / 16
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(16): fn()
    g.replay(); torch.cuda.synchronize()
    e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
    print(name, "eager us", round(1e3 * eager, 1), "graph us", round(1e3 * e0.elapsed_time(e1) / 16, 1), flush=True)
