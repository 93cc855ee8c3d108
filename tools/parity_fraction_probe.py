"""Print the fraction of stored factor entries identical to the oracle's (fp16/bf16 storage),
for the exact (Alg. 1 operation order) and the fast update form, per kernel family / k.
Used to set the low-precision parity bars."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from oracle import pyoracle as po
from paper_conf_hpdc_xietfl17_b200 import mf, synth

HP = dict(lambda_p=0.05, alpha=0.08, beta=0.3)
tiny = synth.tiny(seed=0)
rag = synth.uniform(m=331, n=197, N=12_345, seed=7, mu=0.5, rank=3, noise=0.1, Ntest=777)
cases = [("tiny", 16, dict(schedule="wavefront", workers=8, wf_cols=16), 1)]
for k in (32, 64, 128, 256):
    cases.append(("ragged", k, dict(schedule="wavefront", workers=6, wf_cols=9), 1))
    cases.append(("ragged", k, dict(schedule="hogwild", workers=1), 1))
    cases.append(("ragged", k, dict(schedule="hogwild", workers=1), 2))
for storage in ("fp16", "bf16"):
    for name, k, kw, ep in cases:
        R = tiny if name == "tiny" else rag
        o = po.Oracle(R.m, R.n, k, R.u, R.v, R.r, storage=storage, **HP, **kw)
        for _ in range(ep):
            o.train_epoch()
        Po, Qo = o.factors()
        out = []
        for exact in (True, False):
            g = mf.MF(R.m, R.n, k, storage=storage, exact_order=exact, **HP, **kw)
            g.load(R.u, R.v, R.r)
            for _ in range(ep):
                g.train_epoch()
            Pg, Qg = g.factors()
            mant = 10 if storage == "fp16" else 7
            ulp = max(2.0 ** (np.floor(np.log2(np.abs(X).max())) - mant) for X in (Po, Qo))
            dmax = max(np.abs(Pg - Po).max(), np.abs(Qg - Qo).max()) / ulp
            out.append(f"{'exact' if exact else 'fast'} same P {np.mean(Pg == Po):.4f} Q {np.mean(Qg == Qo):.4f} maxdiff {dmax:.1f} ulp")
            g.close()
        print(storage, name, k, kw["schedule"], f"epochs={ep}", " | ".join(out), flush=True)
