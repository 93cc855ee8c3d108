"""GPU vs oracle on identical Hugewiki-shaped data (small fraction), k = 128, serial orders."""
import sys
sys.path.insert(0, ".")
import numpy as np
from oracle import pyoracle as po
from paper_conf_hpdc_xietfl17_b200 import mf, synth

R = synth.shaped("hugewiki", fraction=0.002, device="cpu")
u, v, r = R.u.numpy(), R.v.numpy(), R.r.numpy()
ut, vt, rt = R.ut.numpy(), R.vt.numpy(), R.rt.numpy()
HP = dict(lambda_p=0.03, alpha=0.08, beta=0.3)
o = po.Oracle(R.m, R.n, 128, u, v, r, **HP)
for kw in (dict(schedule="hogwild", workers=1), dict(schedule="wavefront", workers=64),
           dict(schedule="hogwild", workers=0)):
    g = mf.MF(R.m, R.n, 128, **HP, **kw)
    g.load(u, v, r); g.load(ut, vt, rt, "test")
    cur = []
    for e in range(3):
        g.train_epoch()
        try:
            cur.append(round(g.rmse(), 5))
        except Exception as ex:
            cur.append(str(ex)[:30]); break
    print("GPU", kw, cur, flush=True)
    g.close()
oc = []
for e in range(3):
    o.train_epoch(); oc.append(round(o.rmse(ut, vt, rt), 5))
print("oracle hogwild-serial", oc, flush=True)
