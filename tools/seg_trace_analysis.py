"""Per-tile look-back trace by tile kind (start / seg = a problem start inside the tile / plain):
stage latencies, descriptor round trips and the look-back queue, by distance from the last
problem start.   python tools/seg_trace_analysis.py TRACE.npy N G"""
import numpy as np, sys
N=int(sys.argv[2]); G=int(sys.argv[3])
R=np.load(sys.argv[1]).astype(np.int64)
tiles=R.shape[0]; TILE=8192
t=np.arange(tiles)
r=(t*TILE)%N
nxt=np.where(r==0,N,N-r)
cnt=np.minimum(TILE, G*N - t*TILE)
seg=(nxt<cnt); start=(r==0)
kind=np.where(start,'start',np.where(seg,'seg','plain'))
T=R[:,:5].astype(float)/1e3
print("tiles",tiles,"start",start.sum(),"seg",seg.sum(), "span", (T[:,3].max()-T[:,0].min()))
for k in ('start','seg','plain'):
    m=kind==k
    if m.sum()==0: continue
    print("  %-5s n=%5d ready->A p50 %.2f | A->P p50 %.2f p90 %.2f | RT p50 %.1f p90 %.1f | lbstart-A p50 %.2f | lbdur p50 %.2f | P->written p50 %.2f"%(k,m.sum(),
      np.median(T[m,1]-T[m,0]), np.median(T[m,2]-T[m,1]), np.percentile(T[m,2]-T[m,1],90),
      np.median(R[m,5]), np.percentile(R[m,5],90), np.median(T[m,4]-T[m,1]), np.median(T[m,2]-T[m,4]), np.median(T[m,3]-T[m,2])))
last=-1; d=[]
for i in range(tiles):
    if kind[i]!='plain': last=i
    d.append(i-last)
d=np.array(d); m=kind=='plain'
for dd in range(1,9):
    mm=m&(d==dd)
    if mm.sum(): print("   plain at distance %d: n=%d RT p50 %.1f A->P p50 %.2f lbstart-A %.2f"%(dd,mm.sum(),np.median(R[mm,5]),np.median(T[mm,2]-T[mm,1]),np.median(T[mm,4]-T[mm,1])))
# window readiness vs look-back start for plain tiles
ok=0; bad=0; ex=[]
for i in range(tiles):
    if kind[i]!='plain': continue
    dd=d[i]
    wmax=T[i-dd:i,1].max()   # A (or P-at-A for seg) of tiles between the seg tile and i, incl. seg
    if T[i,4] > wmax + 0.3:
        if R[i,5] > 1: bad+=1; ex.append(i)
        else: ok+=1
print("plain tiles whose window was complete at look-back start: RT==1: %d, RT>1: %d"%(ok,bad))
for i in ex[:5]:
    dd=d[i]
    print(" tile",i,"dist",dd,"lbstart %.2f"%T[i,4],"window A",np.round(T[i-dd:i,1],2),"RT",R[i,5],"P %.2f"%T[i,2])
