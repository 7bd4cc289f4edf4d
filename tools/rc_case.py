"""racecheck / sanitizer driver: one scan shape through one kernel family.

    compute-sanitizer --tool racecheck python tools/rc_case.py N G [algo [param]]
"""
import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import torch, inputs, paper_conf_ipps_dieguezadnm18_b200 as sb
N, G = int(sys.argv[1]), int(sys.argv[2])
algo = sys.argv[3] if len(sys.argv) > 3 else "cascade_cta"
param = int(sys.argv[4]) if len(sys.argv) > 4 else -1
x = torch.empty(N * G, dtype=torch.int32, device="cuda"); inputs.fill_device(x, "i32", 1)
x = x.view(G, N)
for kind in ("inclusive", "exclusive"):
    sb.scan(x, "add", kind, algo=algo, param=param)
torch.cuda.synchronize(); print("done", N, G, algo, param)
