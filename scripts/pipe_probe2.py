"""Probe 2: pipelined host API on a diagonal matrix (trivial kernel)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_dsn_schollbkw16_b200 import encode, inputs as G, NOCHECK, CHECK
from paper_conf_dsn_schollbkw16_b200.abft import PinnedArray
n = 2 * 1024 * 1024
A = G.CSR(np.arange(n + 1, dtype=np.int32), np.arange(n, dtype=np.int32), np.full(n, 2.0), "diag")
h = encode(A)
px, py = PinnedArray(n), PinnedArray(n)
px.a[:] = 1.0
for mode, lab in ((NOCHECK, "diag NOCHECK"), (CHECK, "diag CHECK")):
    h.spmv_host_pipelined([px.a] * 4, [py.a] * 4, mode)
    t0 = time.perf_counter()
    h.spmv_host_pipelined([px.a] * 100, [py.a] * 100, mode)
    print(lab, (time.perf_counter() - t0) / 100 * 1e3, "ms/step")
    t0 = time.perf_counter()
    for _ in range(100):
        h.spmv_host(px.a, py.a, mode)
    print(lab, "sync", (time.perf_counter() - t0) / 100 * 1e3, "ms/step")
