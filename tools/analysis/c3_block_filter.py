"""Offline count (CPU, scipy) on a 1/8-scale C3 graph, degree-relabelled: per BFS level,
the share of probes whose 32/256/1024/4096-id block is entirely visited at the level start
(a coarse visited summary as a probe filter).
  python tools/analysis/c3_block_filter.py"""
import sys, numpy as np, scipy.sparse as sp
sys.path.insert(0,'/root/repo'); import synth
div=8
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
rng=np.random.default_rng(1)
src0=rng.choice(np.nonzero(deg>0)[0])
depth=np.full(n,-1,np.int64); depth[src0]=0; fr=np.array([src0]); L=0
while len(fr):
    vis=(depth>=0)|iso; z=np.nonzero(~vis)[0]; vpre=z[0] if len(z) else n
    idx=A[fr].indices
    tg=idx[idx>=vpre]; dv=depth[tg]
    if len(tg)>1e5:
        s=f'L{L} lists {len(fr)} probes {len(tg)/1e6:.1f}M vis_at_start {np.mean(dv>=0):.3f}'
        for B in [32,256,1024,4096]:
            nb=(n+B-1)//B
            pad=np.ones(nb*B,bool); pad[:n]=vis
            full=pad.reshape(nb,B).all(1)
            s+=f' | B{B}: full-filter {np.mean(full[tg//B]):.3f} (summary {nb/8/1024:.0f} KB at 1/8 scale)'
        print(s,flush=True)
    nxt=np.unique(tg[dv<0]); depth[nxt]=L+1; fr=nxt; L+=1
