import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import torch, inputs, paper_conf_ipps_dieguezadnm18_b200 as sb
N, G = int(sys.argv[1]), int(sys.argv[2])
algo = sys.argv[3] if len(sys.argv) > 3 else "cascade_cta"
x = torch.empty(N * G, dtype=torch.int32, device="cuda"); inputs.fill_device(x, "i32", 1)
x = x.view(G, N)
sb.scan(x, "add", algo=algo); torch.cuda.synchronize(); print("done", N, G, algo)
