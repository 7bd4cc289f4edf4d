"""configs[0] (G = 1, N = 2^20 int32 add) through AUTO: us per call from CUDA-graph replays
of 50 back-to-back calls (bench.py's method), three repetitions."""
import sys; sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
import torch, inputs, paper_conf_ipps_dieguezadnm18_b200 as sb
from bench import device_time
x=torch.empty(1<<20,dtype=torch.int32,device='cuda'); inputs.fill_device(x,'i32',1); y=torch.empty_like(x)
s=torch.cuda.Stream()
for r in range(3): print('c1 us', device_time(lambda: sb.scan(x,'add',out=y,stream=s), s, 50)*1e3, sb.plan(x,y))
