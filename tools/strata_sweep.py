"""Hogwild throughput vs strata grid a and batch f (single GPU)."""
import sys
sys.path.insert(0, ".")
import numpy as np
import torch
from paper_conf_hpdc_xietfl17_b200 import mf, synth

R = synth.shaped("netflix", device="cuda")
cfgs = [dict(grid_a=a, batch_f=f) for a in (1, 8) for f in (256, 512, 1024, 2048, 4096)]
cfgs += [dict(grid_a=2, batch_f=1024), dict(grid_a=4, batch_f=1024)]
for cfg in cfgs:
    kw = dict(storage="fp16", lambda_p=0.05, alpha=0.08, beta=0.3)
    kw.update(cfg)
    g = mf.MF(R.m, R.n, 128, **kw)
    g.load(R.u, R.v, R.r)
    g.load(R.ut, R.vt, R.rt, "test")
    ms = []
    for e in range(6):
        g.train_epoch()
        st = g.stats()
        if e >= 1:
            ms.append(st["sgd_ms"])
    print(cfg, "sgd ms/epoch", round(float(np.mean(ms)), 2), "rmse@6", round(g.rmse(), 5), flush=True)
    g.close()
