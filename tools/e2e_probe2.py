import sys, time, torch, numpy as np
sys.path.insert(0, '.')
import paper_conf_ipps_dieguezadnm18_b200 as sb
for G in (4096, 16384):
    N = 1 << 14
    a = torch.empty(G * N, dtype=torch.int32, pin_memory=True).numpy().reshape(G, N)
    b = torch.empty(G * N, dtype=torch.int32, pin_memory=True).numpy().reshape(G, N)
    a[:] = 1
    sb.scan_host(a, "add", out=b)
    t0 = time.perf_counter()
    for _ in range(5):
        sb.scan_host(a, "add", out=b)
    dt = (time.perf_counter() - t0) / 5
    print("G=%d bytes each way %.0f MB: %.2f ms -> %.1f GB/s each way" % (G, G * N * 4 / 1e6, dt * 1e3, G * N * 4 / dt / 1e9))
# raw pinned copies, one direction at a time and both
n = 1 << 28
h = torch.empty(n, dtype=torch.uint8, pin_memory=True); d = torch.empty(n, dtype=torch.uint8, device="cuda")
h2 = torch.empty(n, dtype=torch.uint8, pin_memory=True); d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for name, fn in [("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h2.copy_(d2, non_blocking=True))]:
    fn(); torch.cuda.synchronize(); t0 = time.perf_counter()
    for _ in range(5): fn()
    torch.cuda.synchronize(); dt = (time.perf_counter() - t0) / 5
    print("%s alone %.1f GB/s" % (name, n / dt / 1e9))
def both():
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
    torch.cuda.synchronize()
both(); t0 = time.perf_counter()
for _ in range(5): both()
dt = (time.perf_counter() - t0) / 5
print("both %.1f GB/s each way" % (n / dt / 1e9))
