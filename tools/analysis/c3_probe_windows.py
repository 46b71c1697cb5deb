"""Offline count (CPU, scipy) on a 1/8-scale C3 graph, degree-relabelled: per BFS level,
the share of probes above the visited prefix that a level-start snapshot of the visited
bits would answer, for id windows of 0.25-4 % of n above the prefix.
  python tools/analysis/c3_probe_windows.py [div]"""
import sys, numpy as np, scipy.sparse as sp, time
sys.path.insert(0,'/root/repo'); import synth
div=int(sys.argv[1]) if len(sys.argv)>1 else 8
cfg=synth.CONFIGS[3]; n=cfg['n']//div; m=cfg['m']//div
n,src,dst=synth.chunglu(n,m,cfg['alpha_src'],cfg['alpha_dst'],cfg['rho'],seed=3)
keep=src!=dst; src=src[keep].astype(np.int64); dst=dst[keep].astype(np.int64)
A=sp.coo_matrix((np.ones(2*len(src),np.int8),(np.r_[src,dst],np.r_[dst,src])),shape=(n,n)).tocsr()
del src,dst
A.sum_duplicates(); A.data[:]=1
deg=np.diff(A.indptr)
order=np.lexsort((np.arange(n),-deg))
A=A[order][:,order].tocsr(); A.sort_indices(); deg=np.diff(A.indptr)
iso=deg==0
nz=np.nonzero(deg>0)[0]
rng=np.random.default_rng(1)
for src0 in rng.choice(nz,3):
  depth=np.full(n,-1,np.int64); depth[src0]=0; fr=np.array([src0]); L=0
  while len(fr):
    vis=(depth>=0)|iso; z=np.nonzero(~vis)[0]; vpre=z[0] if len(z) else n
    idx=A[fr].indices
    tg=idx[idx>=vpre]; dv=depth[tg]
    if len(tg)>1e6:
        s=f'src {src0} L{L} probes {len(tg)/1e6:.1f}M vpre/n {vpre/n:.4f} vis_at_start {np.mean(dv>=0):.3f}'
        for f in [0.0025,0.005,0.01,0.02,0.04]:
            W=int(f*n); s+=f' | w{f}: in {np.mean(tg<vpre+W):.2f} hit {np.mean((tg<vpre+W)&(dv>=0)):.3f}'
        print(s)
    nxt=np.unique(tg[dv<0]); depth[nxt]=L+1; fr=nxt; L+=1
