"""Write oracle reference values for the full-size Hogwild RMSE bar (tests/golden/).

    python tools/oracle_golden.py [--workload netflix] [--epochs 20] [--storage fp16]

Calls ONLY oracle/ (and the shared input generator synth.py, which is counter-based and
therefore yields the same bits on this CPU box as on the GPU box): the plain single-threaded
C oracle runs the batch-Hogwild serial order (Alg. 1, section 5.1 chunk order)
for E epochs on the full Table-2-shaped synthetic set and records the test RMSE after every
epoch, with the data checksum the GPU test re-derives before comparing.  North_star: "Under
Hogwild, test RMSE after 20 epochs must land within 0.5% of the oracle's (fp16 storage: within
1%)".  Takes ~1 h for Netflix (99M ratings x 20 epochs, k = 128, fp16 storage emulated).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import pyoracle as po  # noqa: E402
from paper_conf_hpdc_xietfl17_b200 import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="netflix")
    ap.add_argument("--epochs", type=int, default=20)
    ap.add_argument("--storage", default="fp16")
    ap.add_argument("--k", type=int, default=128)
    ap.add_argument("--fraction", type=float, default=1.0)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    S = synth.SHAPES[a.workload]
    t0 = time.time()
    R = synth.shaped(a.workload, fraction=a.fraction, device="cpu")
    digest = synth.checksum(R)
    print(f"data {a.workload} x{a.fraction}: N={R.N} checksum {digest} ({time.time() - t0:.0f} s)",
          flush=True)
    hp = dict(lambda_p=S["lam"], alpha=S["alpha"], beta=S["beta"], rating_scale=S["rating_scale"])
    u, v, r = (x.numpy() for x in (R.u, R.v, R.r))
    ut, vt, rt = (x.numpy() for x in (R.ut, R.vt, R.rt))
    o = po.Oracle(R.m, R.n, a.k, u, v, r, schedule="hogwild", storage=a.storage, seed=42, **hp)
    curve = [o.rmse(ut, vt, rt)]
    for e in range(a.epochs):
        t1 = time.time()
        o.train_epoch()
        curve.append(o.rmse(ut, vt, rt))
        print(f"epoch {e + 1}: test RMSE {curve[-1]:.6f} ({time.time() - t1:.0f} s)", flush=True)
    out = a.out or os.path.join(ROOT, "tests", "golden",
                                f"{a.workload}_oracle_{a.storage}_hogwild_k{a.k}_e{a.epochs}.json")
    with open(out, "w") as f:
        json.dump({"_source": "tools/oracle_golden.py (oracle/ only): the plain C oracle, batch-"
                              "Hogwild serial order (section 5.1, SURVEY App. A), seed 42, Table 3 "
                              "hyper-parameters; test RMSE after each epoch (index 0 = init)",
                   "workload": a.workload, "fraction": a.fraction, "m": R.m, "n": R.n, "N": R.N,
                   "N_test": R.Ntest, "k": a.k, "storage": a.storage, "schedule": "hogwild",
                   "seed": 42, "hyper": hp, "data_checksum": digest, "epochs": a.epochs,
                   "test_rmse": curve, "seconds": time.time() - t0}, f, indent=1)
    print("wrote", out)


if __name__ == "__main__":
    main()
