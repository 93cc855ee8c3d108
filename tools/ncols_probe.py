"""Hogwild throughput and convergence vs the number of columns n (one GPU, a = 1).

One DSGD block of G GPUs sees only n/a columns at a time (small n "prevents cuMF_SGD from
solving [Netflix, Hugewiki] on multiple GPUs").  This probe fixes m and N per block and varies n,
with the power-law column skew of the shaped sets (a_v = 0.45) and with uniform columns (a_v = 0),
fp16 storage, k = 128, all resident workers.

    python tools/ncols_probe.py [--m 3000000] [--N 24000000]
"""
import argparse
import json
import sys

sys.path.insert(0, ".")
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_hpdc_xietfl17_b200 import mf, synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=3_000_000)
ap.add_argument("--N", type=int, default=24_000_000)
ap.add_argument("--ns", default="1000,2500,5000,10000,20000,40000,160000")
ap.add_argument("--storage", default="fp16")
ap.add_argument("--workers", default="0")
ap.add_argument("--mu", type=float, default=0.0)
ap.add_argument("--epochs", type=int, default=4)
ap.add_argument("--k", type=int, default=128)
args = ap.parse_args()

for n in [int(x) for x in args.ns.split(",")]:
    for a_v in (0.45, 0.0):
        R = synth.powerlaw(args.m, n, args.N, args.N // 100, seed=3, a_v=a_v, mu=args.mu,
                           device="cuda")
        dv = torch.bincount(R.v.long(), minlength=n)
        top = float(dv.max()) / R.N
        for w in [int(x) for x in args.workers.split(",")]:
            g = mf.MF(R.m, R.n, args.k, storage=args.storage, workers=w, lambda_p=0.03, alpha=0.08,
                      beta=0.3, seed=42)
            g.load(R.u, R.v, R.r)
            g.load(R.ut, R.vt, R.rt, "test")
            curve, ms = [round(g.rmse(), 4)], []
            for e in range(args.epochs):
                g.train_epoch()
                st = g.stats()
                ms.append(st["sgd_ms"])
                curve.append(round(g.rmse(), 4))
            print(json.dumps(dict(n=n, a_v=a_v, top_col_share=round(top, 5), workers=st["workers"],
                                  ms=round(float(np.median(ms[1:])), 3),
                                  gups=round(R.N / float(np.median(ms[1:])) / 1e6, 3),
                                  rmse=curve)), flush=True)
            g.close()
        del R
        torch.cuda.empty_cache()
