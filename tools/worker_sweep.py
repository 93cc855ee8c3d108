"""Throughput vs number of parallel workers (paper Figs. 5b, 7a, 11a on B200): batch-Hogwild,
deterministic wavefront and the LIBMF-GPU table-scheduler baseline, Netflix shape, k = 128,
fp16 storage.  Prints one JSON line per point."""
import json
import sys
sys.path.insert(0, ".")
import numpy as np
from paper_conf_hpdc_xietfl17_b200 import mf, synth

R = synth.shaped("netflix", device="cuda")
HP = dict(lambda_p=0.05, alpha=0.08, beta=0.3, storage="fp16")
pts = [("hogwild", w, {}) for w in (64, 256, 1024, 2368, 4736, 9472)]
pts += [("libmf", w, dict(grid_a=2 * w if w <= 512 else 1024)) for w in (16, 64, 128, 256, 512)]
pts += [("wavefront", w, dict(wf_cols=8 * w, cyclic=True)) for w in (128, 256, 512, 1024)]
for sched, w, extra in pts:
    try:
        g = mf.MF(R.m, R.n, 128, schedule=sched, workers=w, **HP, **extra)
        g.load(R.u, R.v, R.r)
        ms = []
        for e in range(3):
            g.train_epoch()
            if e:
                ms.append(g.stats()["sgd_ms"])
        g.close()
        t = float(np.mean(ms))
        print(json.dumps({"schedule": sched, "workers": w, **extra, "sgd_ms": round(t, 2),
                          "G_updates_s": round(R.N / t / 1e6, 3)}), flush=True)
    except Exception as ex:
        print(json.dumps({"schedule": sched, "workers": w, "error": str(ex)[:120]}), flush=True)
