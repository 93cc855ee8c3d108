"""Hugewiki-shaped convergence probe: deterministic wavefront (serial order) vs Hogwild, scaled."""
import sys
sys.path.insert(0, ".")
import math
from paper_conf_hpdc_xietfl17_b200 import mf, synth
for frac in (0.05, 0.3):
    R = synth.shaped("hugewiki", fraction=frac, device="cuda")
    for kw in (dict(schedule="wavefront", workers=512, storage="fp32"),
               dict(schedule="hogwild", workers=256, storage="fp32"),
               dict(schedule="hogwild", workers=0, storage="fp32")):
        g = mf.MF(R.m, R.n, 128, lambda_p=0.03, alpha=0.08, beta=0.3, **kw)
        g.load(R.u, R.v, R.r); g.load(R.ut, R.vt, R.rt, "test")
        curve = []
        for e in range(5):
            g.train_epoch()
            try:
                curve.append(round(g.rmse(), 4))
            except Exception:
                curve.append(float("nan")); break
        P, Q = g.factors()
        print(f"frac={frac} N={R.N} n={R.n}", kw, curve, "max|Q|", float(abs(Q).max()), flush=True)
        g.close()
