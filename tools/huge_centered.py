"""Hugewiki-shaped (full size) with centered ratings (mu = 0): does SGD converge?"""
import sys, time
sys.path.insert(0, ".")
import torch
from paper_conf_hpdc_xietfl17_b200 import mf, synth
S = synth.SHAPES["hugewiki"]
t0 = time.time()
R = synth.powerlaw(S["m"], S["n"], S["N"], S["Ntest"], seed=S["data_seed"], mu=0.0, device="cuda")
print("generated", R.N, round(time.time() - t0, 1), "s", flush=True)
for kw in (dict(storage="fp16"), dict(storage="fp16", workers=1984)):
    t0 = time.time()
    g = mf.MF(R.m, R.n, 128, lambda_p=S["lam"], alpha=S["alpha"], beta=S["beta"], **kw)
    g.load(R.u, R.v, R.r); g.load(R.ut, R.vt, R.rt, "test")
    print("loaded", round(time.time() - t0, 1), "s", "rmse0", round(g.rmse(), 4), flush=True)
    cur, ms = [], []
    for e in range(4):
        g.train_epoch(); st = g.stats(); ms.append(round(st["sgd_ms"], 1))
        cur.append(round(g.rmse(), 4))
    print(kw, "rmse", cur, "sgd ms", ms, "updates/s", round(R.N / (ms[-1] / 1e3) / 1e9, 3), "G", flush=True)
    g.close()
