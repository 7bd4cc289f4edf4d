import sys, torch
sys.path.insert(0, '.')
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
which = sys.argv[1]
N = 1 << 33
x = torch.empty(N, dtype=torch.int32, device="cuda"); inputs.fill_device(x, "i32", 2018); y = torch.empty_like(x)
xv, yv = x.view(1, N), y.view(1, N)
if which == "ours_plain":
    sb.scan(xv, "add", out=yv); torch.cuda.synchronize(); print("ok plain")
elif which == "ours_graph":
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        sb.scan(xv, "add", out=yv)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(3):
            sb.scan(xv, "add", out=yv)
    g.replay(); torch.cuda.synchronize(); print("ok graph")
elif which == "torch":
    torch.cumsum(xv, dim=1, dtype=torch.int32, out=yv); torch.cuda.synchronize(); print("ok torch")
if which == "torch_graph":
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        torch.cumsum(xv, dim=1, dtype=torch.int32, out=yv)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(3):
            torch.cumsum(xv, dim=1, dtype=torch.int32, out=yv)
    g.replay(); torch.cuda.synchronize(); print("ok torch graph")
if which == "sweep_order":
    sys.argv = ["paper_sweep.py", "g1", "33", "33"]
    sys.path.insert(0, "tools")
    import paper_sweep
    paper_sweep.main()
