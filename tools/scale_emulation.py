"""Multi-GPU DSGD-strata scaling, emulated on ONE B200 (this environment gives one GPU per call).

With the fixed a x a = 8 x 8 grid (R21), in sub-epoch j rank g of G trains the a/G
blocks of row segments [g a/G, (g+1) a/G).  Running world = 1 with grid_a = 8 and
launch_blocks = a/G makes every SGD launch exactly one rank's sub-epoch work (same blocks, same
chunk order, same kernel); the blocks of a stratum touch disjoint P and Q rows, so the result is
the same as the G-GPU run.  The emulated G-GPU epoch is

    T_G = sum_j max_g t(j, g)  +  a * t_comm

with t(j, g) the measured device time of launch (j, g) and t_comm the Q-rotation step: one
ncclSend/ncclRecv pair of ceil(n/a) k S bytes per rank, estimated as 20 us latency + bytes at
the measured 770 GB/s NVLink peer bandwidth (B200_PROFILING.md).  updates/s = N / T_G.

    python tools/scale_emulation.py [--workload hugewiki] [--fraction 1.0] [--epochs 3]
"""
import argparse
import json
import sys

sys.path.insert(0, ".")
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_hpdc_xietfl17_b200 import mf, synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="netflix")
ap.add_argument("--fraction", type=float, default=1.0)
ap.add_argument("--epochs", type=int, default=3)
ap.add_argument("--storage", default="fp16")
ap.add_argument("--batch-f", type=int, default=256)
ap.add_argument("--out", default=None)
ap.add_argument("--gs", default="1,2,4,8", help="GPU counts to emulate")
ap.add_argument("--workers", default="0", help="comma list of Hogwild worker counts (0 = all resident)")
ap.add_argument("--no-base", action="store_true")
ap.add_argument("--group-cols", action="store_true", help="column-grouped batches (R24) in the G runs")
args = ap.parse_args()

s = synth.SHAPES[args.workload]
R = synth.shaped(args.workload, fraction=args.fraction, device="cuda")
hp = dict(lambda_p=s["lam"], alpha=s["alpha"], beta=s["beta"], rating_scale=s["rating_scale"])
K, A = 128, 8
S = 2 if args.storage != "fp32" else 4
msg = -(-R.n // A) * K * S
t_comm = 20e-3 + msg / 770e9 * 1e3          # ms per sub-epoch


def run(**kw):
    g = mf.MF(R.m, R.n, K, storage=args.storage, seed=42, **hp, **kw)
    g.load(R.u, R.v, R.r)
    g.load(R.ut, R.vt, R.rt, "test")
    g.train_epoch()                          # warm-up
    per = []
    for _ in range(args.epochs):
        g.train_epoch()
        per.append(g.launch_ms())
    rmse = g.rmse()
    upd = g.stats()["updates"]
    g.close()
    del g
    torch.cuda.empty_cache()                 # the next ctx needs the 37 GB slot array again
    return np.array(per), rmse, upd


rows = []
t1 = float("nan")
if not args.no_base:
    base, rmse1, upd = run(grid_a=1, batch_f=256)
    t1 = float(base.sum(1).mean())
    rows.append(dict(G=1, grid="a=1 f=256", ms_epoch=t1, gups=upd / t1 / 1e6, rmse=rmse1))
    print(json.dumps(rows[-1]), flush=True)
for G, W in [(int(g), int(w)) for g in args.gs.split(",") for w in args.workers.split(",")]:
    per, rmse, upd = run(grid_a=A, batch_f=args.batch_f, launch_blocks=A // G, workers=W,
                         group_cols=args.group_cols)
    assert per.shape[1] == A * G, per.shape
    t = per.reshape(per.shape[0], A, G)                     # [epoch, sub-epoch j, rank g]
    comp = float(t.max(2).sum(1).mean())
    imb = float((t.max(2) / t.mean(2)).mean())
    tg = comp + (A * t_comm if G > 1 else 0.0)
    rows.append(dict(G=G, workers=W, grid=f"a={A} f={args.batch_f} blocks/launch={A // G}"
                     + (" grouped" if args.group_cols else ""),
                     compute_ms=comp, comm_ms_est=A * t_comm if G > 1 else 0.0, ms_epoch=tg,
                     gups=upd / tg / 1e6, per_gpu_gups=upd / tg / 1e6 / G,
                     efficiency_vs_a1=(upd / tg) / (G * upd / t1), load_imbalance=imb, rmse=rmse))
    print(json.dumps(rows[-1]), flush=True)
if args.out:
    with open(args.out, "w") as f:
        json.dump(dict(workload=args.workload, fraction=args.fraction, N=R.N, m=R.m, n=R.n,
                       storage=args.storage, t_comm_ms=t_comm, rows=rows), f, indent=1)
