import torch, time
n = 2 * 1024 * 1024
xh = torch.randn(n, dtype=torch.float64).pin_memory()
yh = torch.empty(n, dtype=torch.float64).pin_memory()
xd = torch.empty(n, dtype=torch.float64, device="cuda")
yd = torch.randn(n, dtype=torch.float64, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def t(fn, k=50):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    for _ in range(k): fn()
    torch.cuda.synchronize(); return (time.perf_counter() - t0) / k * 1e3
def h2d():
    with torch.cuda.stream(s1): xd.copy_(xh, non_blocking=True)
def d2h():
    with torch.cuda.stream(s2): yh.copy_(yd, non_blocking=True)
def both():
    h2d(); d2h()
for f in (h2d, d2h, both): t(f, 5)
print("h2d ms", t(h2d), "d2h ms", t(d2h), "both ms", t(both))
