import sys; sys.path.insert(0,'.')
import numpy as np
from paper_conf_hpdc_xietfl17_b200 import mf
rng=np.random.default_rng(0); N=300000; m,n=400000,17000
for st in ("fp32","fp16"):
  for lb in (16,32):
    g=mf.MF(m,n,128,storage=st,schedule="wavefront",workers=1,wf_cols=1,lane_bytes=lb,alpha=0.001,beta=0.0)
    g.load(rng.integers(0,m,N).astype(np.int32), np.zeros(N,np.int32), np.ones(N,np.float32))
    g.train_epoch(); g.train_epoch(); s=g.stats(); g.close()
    print(st, lb, "lanes", s["lanes"], "q-chain ns/upd", round(1e6*s["sgd_ms"]/N,1))
