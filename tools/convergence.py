"""Hogwild concurrency vs convergence study (paper section 7.5; E4/E10 analogues).

Runs the GPU path with several worker counts / schedules and prints test RMSE per epoch as
JSON lines; for small sets also the serial oracle's RMSE (same seeded inputs).
    python tools/convergence.py --set tiny|powerlaw|netflix [--epochs 20] [--oracle]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_hpdc_xietfl17_b200 import mf, synth  # noqa: E402


def get_set(name):
    if name == "tiny":
        R = synth.tiny(seed=0)
        return R, dict(lambda_p=0.05, alpha=0.08, beta=0.3), 16
    if name == "powerlaw":
        R = synth.powerlaw(4000, 900, 200_000, 20_000, seed=5, rank=8, mu=3.6, noise=0.5)
        R = synth.Ratings(R.m, R.n, R.u.numpy(), R.v.numpy(), R.r.numpy(), R.ut.numpy(),
                          R.vt.numpy(), R.rt.numpy())
        return R, dict(lambda_p=0.05, alpha=0.08, beta=0.3), 32
    s = synth.SHAPES[name]
    R = synth.shaped(name, device="cuda")
    return R, dict(lambda_p=s["lam"], alpha=s["alpha"], beta=s["beta"],
                   rating_scale=s["rating_scale"]), 128


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--set", default="tiny")
    ap.add_argument("--epochs", type=int, default=20)
    ap.add_argument("--oracle", action="store_true")
    ap.add_argument("--storage", default="fp32")
    ap.add_argument("--runs", default="")
    a = ap.parse_args()
    R, hp, k = get_set(a.set)
    runs = [json.loads(x) for x in a.runs.split(";")] if a.runs else [
        {"schedule": "hogwild", "workers": w} for w in (1, 8, 32, 128, 0)]
    for run in runs:
        g = mf.MF(R.m, R.n, k, storage=a.storage, **hp, **run)
        g.load(R.u, R.v, R.r)
        g.load(R.ut, R.vt, R.rt, "test")
        curve, ms = [], []
        for _ in range(a.epochs):
            g.train_epoch()
            st = g.stats()
            ms.append(st["epoch_ms"])
            curve.append(round(g.rmse(), 6))
        print(json.dumps({"set": a.set, "storage": a.storage, **run, "eff_workers": st["workers"],
                          "epoch_ms": round(float(np.median(ms)), 3), "rmse": curve}), flush=True)
        g.close()
    if a.oracle:
        from oracle import pyoracle as po
        o = po.Oracle(R.m, R.n, k, R.u, R.v, R.r, storage=a.storage, **hp)
        curve = []
        t0 = time.time()
        for _ in range(a.epochs):
            o.train_epoch()
            curve.append(round(o.rmse(R.ut, R.vt, R.rt), 6))
        print(json.dumps({"set": a.set, "storage": a.storage, "oracle": "hogwild-serial",
                          "sec": round(time.time() - t0, 1), "rmse": curve}), flush=True)


if __name__ == "__main__":
    main()
