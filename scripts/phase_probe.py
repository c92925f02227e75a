"""Timing experiment 8 (ABFT_LIB=libabft_e8.so): per-phase SM cycles of the
SHORT k_stream consumers, averaged per consumer step (one group per warp).
Phases: 0 wait full, 1 phase A (next group's loads / gathers issued),
2 finish + release (3 + 4 + 5 + arrive), 3 y (products, tree, store),
4 C pass (position stores, t1 products, tree), 5 reduce-scatter + test."""
import ctypes as C
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_dsn_schollbkw16_b200 import CHECK, encode, inputs as G, lib

n = int(sys.argv[1]) if len(sys.argv) > 1 else 128
A = G.laplacian_3d_7pt(n)
h = encode(A, 32)
x = torch.from_numpy(G.uniform_vector(A.n, 42)).cuda()
y = torch.empty_like(x)
L = lib()
buf = (C.c_ulonglong * 8)()
for mode, name in ((CHECK, "protected"), (0, "plain")):
    for _ in range(20):
        h.spmv(x, y, mode=mode)
    torch.cuda.synchronize()
    L.abft_debug_phases(buf)
    reps = 200
    for _ in range(reps):
        h.spmv(x, y, mode=mode)
    torch.cuda.synchronize()
    L.abft_debug_phases(buf)
    v = np.array(list(buf), dtype=np.float64)
    steps = max(v[6], 1)
    names = ["wait", "phaseA", "finish+rel", "y", "Cpass", "bfly+test"]
    print(name, f"steps/call {steps / reps:.0f}", " ".join(f"{k}={v[i] / steps:.0f}" for i, k in enumerate(names)))
