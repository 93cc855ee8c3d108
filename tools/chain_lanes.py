"""Serial q-chain latency (ns per update, one worker) of the ring kernel per lane geometry."""
import sys

import numpy as np

sys.path.insert(0, ".")
from paper_conf_hpdc_xietfl17_b200 import mf  # noqa: E402

rng = np.random.default_rng(0)
N, m, n = 300_000, 400_000, 17_000
for st in ("fp32", "fp16"):
    for k in ((128,) if st == "fp32" else (128, 256)):
        for lb in (16, 32, 64):
            for chain in ("q", "none"):
                u = rng.integers(0, m, N).astype(np.int32)
                v = np.zeros(N, np.int32) if chain == "q" else rng.integers(0, n, N).astype(np.int32)
                g = mf.MF(m, n, k, storage=st, schedule="wavefront", workers=1, wf_cols=1,
                          lane_bytes=lb, alpha=0.001, beta=0.0)
                g.load(u, v, np.ones(N, np.float32))
                g.train_epoch()
                g.train_epoch()
                s = g.stats()
                g.close()
                print(st, "k", k, "lane_bytes", lb, "lanes", s["lanes"], chain + "-chain ns/upd",
                      round(1e6 * s["sgd_ms"] / N, 1), flush=True)
