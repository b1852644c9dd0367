#!/usr/bin/env python
"""Source-row reuse vs in-block options for 2/3/4-layer blocking on the oracle's GPT tables (analysis for
profiles/r02b_step_bounds.md; oracle only):  python scripts/blocking_reuse.py <candidate j>"""
import json, sys, numpy as np
sys.path.insert(0, __import__('os').path.dirname(__import__('os').path.dirname(__import__('os').path.abspath(__file__))))
import oracle, chaingen
cfg=json.load(open(__import__('os').path.join(sys.path[0], 'configs', 'gpt.json')))
ch=chaingen.gpt(); P=cfg['P']; M=cfg['M']; beta=cfg['beta']; nm=cfg['n_mem']; nv=cfg['n_delay']; nc=cfg['n_periods']
pr=oracle.prep(ch,P,beta); lb,ub=pr['lb'],pr['ub']; Up=pr['Up']; L=len(ch['uF']); SC=pr['SC']
W=np.array(ch['W'],dtype=np.int64); Wp=np.concatenate([[0],np.cumsum(W)])
j=int(sys.argv[1]); tau = lb + j*((ub-lb)/(nc-1)); dV=(Up[L]+SC)/(nv-1)
A,_,cu=oracle.table(ch,P,M,beta,nm,nv,0,tau,with_arg=False)
fin = np.isfinite(A).any(axis=(1,3))
def win(l): return [k for k in range(1,l+1) if Up[l]-Up[k-1]<=tau and 3*(Wp[l]-Wp[k-1])<=M]
for B,VB in [(2,4),(3,3),(4,2)]:
    tot_rows=0; tot_ent=0; inblock=0
    for l0 in [41,121,201]:
        shifts=[int(np.rint((Up[l0+i]-Up[l0])/dV)) for i in range(B)]
        for vt in range(-(20//VB), nv//VB+1):
            rows=[(l0+i, vt*VB - shifts[i] + r) for i in range(B) for r in range(VB)]
            ents=set()
            for (lr,v) in rows:
                if v<0 or v>=nv: continue
                for k in win(lr):
                    g,nf,d,vn=oracle.transition(ch,P,M,beta,nm,nv,0,tau,k,lr,v)
                    if vn<0 or vn>nv-1: continue
                    if not nf and d>nm-1: continue
                    if not fin[k-1][vn]: continue
                    if k > l0: inblock+=1; continue
                    tot_rows+=1; ents.add((k,vn))
            tot_ent+=len(ents)
    print('B',B,'VB',VB,'row-visits(shared part)',tot_rows,'entries',tot_ent,'reuse',tot_rows/tot_ent,'in-block visits',inblock, flush=True)
