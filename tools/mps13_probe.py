"""Scan-MPS at W = 1, n = 13 (G = 32768 problems of 8192): the elements-mode call with the
fused-exchange communicator of one rank, ms per call from events around 10 calls (for an
ncu launch list of the pipeline's kernels)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
from paper_conf_ipps_dieguezadnm18_b200 import multi
n=13; N=1<<n; G=(1<<28)//N
x=torch.empty(G*N,dtype=torch.int32,device="cuda"); inputs.fill_device(x,"i32",3); x=x.view(G,N); y=torch.empty_like(x)
c=multi.PeerComm.loopback(1,G)[0]
for _ in range(3): multi.scan_multi(x,"add","inclusive",mode="elements",out=y,backend="peer",comm=c)
torch.cuda.synchronize()
e0,e1=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10): multi.scan_multi(x,"add","inclusive",mode="elements",out=y,backend="peer",comm=c)
e1.record(); torch.cuda.synchronize(); print("ms per call", e0.elapsed_time(e1)/10)
c.close()
