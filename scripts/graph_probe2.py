"""Probe: which part of a sharded-PCG iteration loses time under CUDA-graph
replay (N = 1, 192^3)?  Eager vs graph for 16 repetitions of (a) the
protected distributed SpMV, (b) the PCG vector phases + combines."""
import torch

from paper_conf_dsn_schollbkw16_b200 import inputs as G
from paper_conf_dsn_schollbkw16_b200 import parallel as PL
from paper_conf_dsn_schollbkw16_b200.abft import PCG_PHASE_DOT, PCG_PHASE_P, PCG_PHASE_UPDATE

n3 = 192
rows = G.stencil_rows("7pt", n3, n3, n3, 0, n3)
sh = PL.make_shard(rows, 0, n3 ** 3, 0, 1, [(0, n3 ** 3)])
d = PL.DistSpmv(sh)


class Solo:
    def gather_partials(self, p, o):
        o.copy_(p)

    def halo(self, a, b):
        pass


c = Solo()
d.own().copy_(torch.from_numpy(G.uniform_vector(sh.n, 43)))
b = d.plain(c).clone()
x = torch.from_numpy(G.uniform_vector(sh.n, 44)).cuda()
p = PL.DistPcg(d, True)
p.begin(b, x, sh.n, max_iter=10 ** 9, tol=0.0)


def spmv():
    part = p.spmv_local(c)
    c.gather_partials(part, d.parts)
    p.spmv_finish()


def vec(j):
    for ph in (PCG_PHASE_DOT, PCG_PHASE_UPDATE):
        p.local(ph, j)
        c.gather_partials(p.send, p.recv)
        p.combine(ph, j)
    p.local(PCG_PHASE_P, j)


cases = {"spmv": lambda j: spmv(), "vector": vec, "both": lambda j: (spmv(), vec(j))}
for name, fn in cases.items():
    for j in range(1, 4):
        fn(j)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for j in range(1, 17):
        fn(j)
    e1.record()
    torch.cuda.synchronize()
    eager = e0.elapsed_time(e1) / 16
    g = torch.cuda.CUDAGraph()
    cs = torch.cuda.Stream()
    cs.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(cs):
        g.capture_begin()
        for j in range(1, 17):
            fn(j)
        g.capture_end()
    torch.cuda.current_stream().wait_stream(cs)
    g.replay()
    torch.cuda.synchronize()
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    print(name, "eager us/iter", round(1e3 * eager, 1), "graph us/iter",
          round(1e3 * e0.elapsed_time(e1) / 16, 1), flush=True)
