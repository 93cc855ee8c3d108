"""Small runs of every kernel family for compute-sanitizer.

    compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_case.py all
    compute-sanitizer --tool racecheck --error-exitcode 9 python tools/sanitize_case.py det

Seeded uniform ratings with duplicates (numpy), m = 301, n = 157, 6,000 train / 500 test
ratings; each case trains 1-2 epochs, evaluates RMSE and reads the factors back.  'det' runs the
deterministic (wavefront) kernels only: they must be race-free; Hogwild races on P/Q by design.
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpdc_xietfl17_b200 import mf  # noqa: E402

HP = dict(lambda_p=0.05, alpha=0.08, beta=0.3)
DET = [
    dict(k=128, storage="fp32", schedule="wavefront", workers=6, wf_cols=9),                # 16-B ring
    dict(k=128, storage="fp16", schedule="wavefront", workers=6, wf_cols=9, cyclic=True),   # 8-B ring
    dict(k=64, storage="fp16", schedule="wavefront", workers=5, wf_cols=7, grid_a=4),       # 4-B ring
    dict(k=16, storage="fp32", schedule="wavefront", workers=4, wf_cols=8),                 # 16-lane ring
    dict(k=32, storage="fp32", schedule="wavefront", workers=4, wf_cols=8, wf_kernel=2),    # register
    dict(k=32, storage="fp32", schedule="wavefront", workers=4, wf_cols=8, lr_rule="adagrad"),
    dict(k=128, storage="fp16", schedule="wavefront", workers=6, wf_cols=9, exact_order=True,
         check_owners=True),                                                                # exact form + checker
    dict(k=64, storage="fp32", schedule="wavefront", workers=4, wf_cols=6, grid_a=4, staged=2,
         stage_chunk=1000),                                                                 # P out of core
]
RACY = [
    dict(k=16, storage="fp32", schedule="hogwild"),
    dict(k=128, storage="fp16", schedule="hogwild", grid_a=4, batch_f=64, launch_blocks=2),
    dict(k=128, storage="bf16", schedule="hogwild", staged=True, grid_a=2),
    dict(k=64, storage="fp32", schedule="libmf", grid_a=4),
    dict(k=32, storage="fp32", schedule="hogwild", lr_rule="adagrad"),
    dict(k=128, storage="fp16", schedule="hogwild", rating_stage=1, batch_f=128),      # TMA rating stream
    dict(k=128, storage="fp16", schedule="hogwild", group_cols=True, batch_f=512),     # grouped batches
    dict(k=32, storage="fp32", schedule="hogwild", grid_a=4, batch_f=64, staged=True,
         stage_chunk=1500),                                                             # chunked out-of-core load
    dict(k=128, storage="bf16", schedule="hogwild", grid_a=4, batch_f=64, staged=2),   # P out of core
    dict(k=16, storage="fp16", schedule="hogwild", exact_order=True),
]


def data(seed=3, m=301, n=157, N=6000, Nt=500):
    rng = np.random.default_rng(seed)
    u = rng.integers(0, m, N + Nt).astype(np.int32)
    v = rng.integers(0, n, N + Nt).astype(np.int32)
    r = (0.5 + rng.standard_normal(N + Nt) * 0.3).astype(np.float32)
    return m, n, (u[:N], v[:N], r[:N]), (u[N:], v[N:], r[N:])


def run(case):
    m, n, tr, te = data()
    kw = dict(case)
    k = kw.pop("k")
    g = mf.MF(m, n, k, allocator="none", **HP, **kw)
    g.load(*tr)
    g.load(*te, set="test")
    for _ in range(2):
        g.train_epoch()
    rm = g.rmse()
    P, Q = g.factors()
    g.close()
    assert np.isfinite(rm) and np.isfinite(P).all() and np.isfinite(Q).all(), case
    print("ok", case, round(rm, 5), flush=True)


# shared-memory rings of the Hogwild kernels (TMA rating stream), at 1 worker so that the global
# P/Q accesses do not race by design either: racecheck then checks the smem ring protocol
SMEM = [
    dict(k=128, storage="fp16", schedule="hogwild", rating_stage=1, batch_f=128, workers=1),
    dict(k=64, storage="fp32", schedule="hogwild", rating_stage=1, batch_f=64, workers=1, grid_a=2),
]

if __name__ == "__main__":
    which = sys.argv[1] if len(sys.argv) > 1 else "all"
    cases = {"all": DET + RACY, "det": DET, "smem": SMEM}[which]
    for c in cases:
        run(c)
