"""Serial update latency of the deterministic kernels (one worker, one sub-block):
independent samples (random u, v) vs a fully dependent q-chain (every rating in ONE column, so
sample j+1 needs q'_j) vs a dependent p-chain (one row).  ns per update = sgd time / N."""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_hpdc_xietfl17_b200 import mf  # noqa: E402


def run(m, n, u, v, storage, wfk, k=128):
    g = mf.MF(m, n, k, storage=storage, schedule="wavefront", workers=1, wf_cols=1, wf_kernel=wfk,
              alpha=0.001, beta=0.0, lambda_p=0.05)
    r = np.ones(len(u), np.float32)
    g.load(u, v, r)
    g.train_epoch()
    g.train_epoch()
    st = g.stats()
    g.close()
    return 1e6 * st["sgd_ms"] / len(u)


rng = np.random.default_rng(0)
N = 300_000
out = {}
for storage in ("fp32", "fp16"):
    for wfk in (1, 2):
        m, n = 400_000, 17_000
        ind = run(m, n, rng.integers(0, m, N).astype(np.int32), rng.integers(0, n, N).astype(np.int32), storage, wfk)
        qch = run(m, n, rng.integers(0, m, N).astype(np.int32), np.zeros(N, np.int32), storage, wfk)
        pch = run(m, n, np.zeros(N, np.int32), rng.integers(0, n, N).astype(np.int32), storage, wfk)
        out[f"{storage}/wf_kernel={wfk}"] = dict(independent_ns=round(ind, 1), q_chain_ns=round(qch, 1),
                                                  p_chain_ns=round(pch, 1))
        print(storage, wfk, out[f"{storage}/wf_kernel={wfk}"], flush=True)
json.dump(out, open("gpurun_out/chain_latency.json", "w"), indent=1)
