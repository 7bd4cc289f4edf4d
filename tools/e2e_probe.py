"""Time the host-buffer path (scan_batch_host) on the configs[1] step; the staging piece
and slot count come from SCANB200_HOST_PIECE / SCANB200_HOST_SLOTS."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
G, N = 4096, 1 << 14
a = torch.empty(G * N, dtype=torch.int32, pin_memory=True).numpy()
a[:] = inputs.generate("i32", G * N, 1)
o = torch.empty(G * N, dtype=torch.int32, pin_memory=True).numpy()
x, y = a.reshape(G, N), o.reshape(G, N)
sb.scan_host(x, "add", out=y)
t0 = time.perf_counter()
for _ in range(8):
    sb.scan_host(x, "add", out=y)
dt = (time.perf_counter() - t0) / 8
print("piece=%s slots=%s  %.2f ms/scan  %.2f Gelem/s  %.1f GB/s each way" % (
    os.environ.get("SCANB200_HOST_PIECE"), os.environ.get("SCANB200_HOST_SLOTS"), dt * 1e3, G * N / dt / 1e9,
    G * N * 4 / dt / 1e9))
