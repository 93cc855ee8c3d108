"""CPU emulation of the two SGD update forms' operation order.

Replays the oracle's exact execution order (export "order") on the tiny set with fp16 storage
and evaluates each update three ways in numpy float32 (fma emulated in float64): 'seq' = the
oracle's own order (must reproduce the oracle bit for bit: a check of the emulation),
'literal' = the paper's operation order with the kernel's lane-partial + butterfly dot
(k_wavefront, L = 4), 'kernel' = the fast 2-op form with that dot.  Prints the fraction of
stored entries identical to the oracle's after one epoch -- the arithmetic's own prediction of
the GPU's fraction (tools/parity_fraction_probe.py measures the GPU: 0.9999 / 0.8976, equal).
Test infrastructure: reads only oracle/ and synth.
"""
import os, sys
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from oracle import pyoracle as po
from paper_conf_hpdc_xietfl17_b200 import synth
f32=np.float32
def fma(a,b,c): return f32(np.float64(a)*np.float64(b)+np.float64(c))
R=synth.tiny(seed=0); k=16
kw=dict(schedule="wavefront",workers=8,wf_cols=16,lambda_p=0.05,alpha=0.08,beta=0.3,storage="fp16")
o=po.Oracle(R.m,R.n,k,R.u,R.v,R.r,**kw)
order=o.export("order",0); perm=o.export("perm")
P0,Q0=o.factors()
o.train_epoch(); Po,Qo=o.factors()
g=f32(po.lib().or_gamma(0.08,0.3,0)); lp=f32(0.05)
def rnd(x): return x.astype(np.float16).astype(np.float32)
def run(variant):
    P=P0.copy(); Q=Q0.copy()
    L=4; VEC=k//L
    for j in order:
        i=perm[j]; u=R.u[i]; v=R.v[i]; r=f32(R.r[i])
        p=P[u].copy(); q=Q[v].copy()
        if variant=='seq':
            acc=f32(0)
            for d in range(k): acc=f32(acc+f32(p[d]*q[d]))
        else:
            parts=[]
            for l in range(L):
                ax=f32(0); ay=f32(0)
                for e in range(0,VEC,2):
                    ax=fma(p[l*VEC+e],q[l*VEC+e],ax); ay=fma(p[l*VEC+e+1],q[l*VEC+e+1],ay)
                parts.append(f32(ax+ay))
            # butterfly xor 2 then xor1 (lane0 view)
            s=[f32(parts[l]+parts[l^2]) for l in range(L)]
            acc=f32(s[0]+s[1])
        if variant in('kernel',):
            ge=fma(-g,acc,f32(g*r)); cp=f32(f32(1)-f32(g*lp))
            pn=np.array([fma(ge,q[d],f32(cp*p[d])) for d in range(k)],f32)
            qn=np.array([fma(ge,p[d],f32(cp*q[d])) for d in range(k)],f32)
        else:
            err=f32(r-acc)
            pn=np.array([f32(p[d]+f32(g*f32(f32(err*q[d])-f32(lp*p[d])))) for d in range(k)],f32)
            qn=np.array([f32(q[d]+f32(g*f32(f32(err*p[d])-f32(lp*q[d])))) for d in range(k)],f32)
        P[u]=rnd(pn); Q[v]=rnd(qn)
    return P,Q
for var in ('seq','literal','kernel'):
    P,Q=run(var)
    print(var, 'P same %.4f Q same %.4f'%((P==Po).mean(),(Q==Qo).mean()), 'maxdiff',np.abs(P-Po).max(),np.abs(Q-Qo).max())
