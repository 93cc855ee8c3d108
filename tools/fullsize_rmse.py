"""Print the 20-epoch test RMSE of the bench configuration (fp16 Hogwild, all resident workers),
the grouped-batch and a x 1 row-block variants and the fp16 deterministic wavefront on the full Netflix-shaped set,
next to the oracle's own 20-epoch run (tests/golden/netflix_oracle_fp16_hogwild_k128_e20.json)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_hpdc_xietfl17_b200 import mf, synth  # noqa: E402

S = synth.SHAPES["netflix"]
HP = dict(lambda_p=S["lam"], alpha=S["alpha"], beta=S["beta"])
R = synth.shaped("netflix", device="cuda")
gold = json.load(open(os.path.join(ROOT, "tests", "golden", "netflix_oracle_fp16_hogwild_k128_e20.json")))
print("checksum", synth.checksum(R), "golden", gold["data_checksum"])
runs = {"hogwild": dict(schedule="hogwild"),
        "hogwild-grouped-f1024": dict(schedule="hogwild", group_cols=True, batch_f=1024),
        "hogwild-rowblocks-auto": dict(schedule="hogwild", grid_cols=1),
        "hogwild-rowblocks-2x1": dict(schedule="hogwild", grid_cols=1, grid_a=2),
        "wavefront-fp16-cyclic": dict(schedule="wavefront", workers=888, wf_cols=7680, cyclic=True)}
out = {}
for name, kw in runs.items():
    g = mf.MF(R.m, R.n, 128, storage="fp16", seed=42, **HP, **kw)
    g.load(R.u, R.v, R.r)
    g.load(R.ut, R.vt, R.rt, "test")
    curve = []
    for _ in range(20):
        g.train_epoch()
        curve.append(g.rmse())
    out[name] = curve
    g.close()
    ro = gold["test_rmse"][20]
    print(f"{name}: epoch 20 test RMSE {curve[-1]:.6f}  oracle {ro:.6f}  rel {(curve[-1] - ro) / ro:+.4%}")
print(json.dumps({"oracle": gold["test_rmse"][1:], **out}))
