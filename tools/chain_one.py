"""One single-worker q-chain wavefront run (fp32, k=128) for ncu source-level stall capture."""
import sys

import numpy as np

sys.path.insert(0, ".")
from paper_conf_hpdc_xietfl17_b200 import mf  # noqa: E402

st = sys.argv[1] if len(sys.argv) > 1 else "fp32"
rng = np.random.default_rng(0)
N, m, n = 300_000, 400_000, 17_000
g = mf.MF(m, n, 128, storage=st, schedule="wavefront", workers=1, wf_cols=1, alpha=0.001, beta=0.0)
g.load(rng.integers(0, m, N).astype(np.int32), np.zeros(N, np.int32), np.ones(N, np.float32))
g.train_epoch()
g.train_epoch()
print("ns/upd", 1e6 * g.stats()["sgd_ms"] / N)
