import os, sys, json
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo")); sys.path.insert(0, os.path.join(os.environ.get("GRAFT_REPO_ROOT", "/root/repo"), "tools"))
import torch, inputs, paper_conf_ipps_dieguezadnm18_b200 as sb
peak = json.load(open(os.path.join(os.environ.get("GRAFT_REPO_ROOT", "/root/repo"), "MEASURED_PEAKS.json")))["hbm_gbs"]
T = 1 << 28
x = torch.empty(T, dtype=torch.int32, device="cuda"); inputs.fill_device(x, "i32", 5); y = torch.empty_like(x)
def ms(f, reps=10):
    for _ in range(3): f()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); a.record()
    for _ in range(reps): f()
    b.record(); torch.cuda.synchronize(); return a.elapsed_time(b) / reps
for rep in range(2):
    for n in (11, 12, 13):
        N = 1 << n; xv, yv = x.view(T // N, N), y.view(T // N, N)
        r = {"n": n}
        for algo in ("cascade_cta", "cascade_warp", "packed_warp"):
            r[algo] = round(8 * T / (ms(lambda: sb.scan(xv, "add", out=yv, algo=algo)) * 1e-3) / 1e9 / peak, 3)
        print(json.dumps(r), flush=True)
