"""Run bench.py over a list of configurations and write a markdown table (profiles/ evidence).

    python tools/sweep.py --name r01_sweep [--set kprec|yahoo|all]
Each row is one `bench.py` run (its own process, device-timed epochs, fresh data).
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SETS = {
    "kprec": [dict(workload="netflix", k=k, storage=s) for k in (32, 64, 128, 256)
              for s in ("fp32", "fp16", "bf16")],
    # configs[4] with the best Hogwild configuration: a x 1 row blocks (R27) + grouped batches (R24)
    "kprec_best": [{"workload": "netflix", "k": k, "storage": s, "grid-cols": 1, "group-cols": True,
                    "batch-f": 1024} for k in (32, 64, 128, 256) for s in ("fp32", "fp16", "bf16")],
    # configs[2] at HEAD: Yahoo-shaped batch-Hogwild (plain, a x 1 rows, rows + grouped) vs wavefront
    "yahoo3": [dict(workload="yahoo", storage="fp16"), dict(workload="yahoo", storage="fp32"),
               {"workload": "yahoo", "storage": "fp16", "grid-cols": 1},
               {"workload": "yahoo", "storage": "fp16", "grid-cols": 1, "group-cols": True, "batch-f": 1024},
               {"workload": "yahoo", "storage": "fp32", "grid-cols": 1},
               dict(workload="yahoo", storage="fp32", schedule="wavefront", workers=888,
                    **{"wf-cols": 15360}, cyclic=True),
               dict(workload="yahoo", storage="fp16", schedule="wavefront", workers=888,
                    **{"wf-cols": 15360}, cyclic=True)],
    # the deterministic configuration of bench.py over k and storage, and the Yahoo shape
    "det": [dict(workload="netflix", k=k, storage=s, schedule="wavefront", workers=888,
                 **{"wf-cols": 7680}, cyclic=True)
            for k in (32, 64, 128, 256) for s in ("fp32", "fp16", "bf16")],
    "yahoo2": [dict(workload="yahoo", storage="fp16"), dict(workload="yahoo", storage="fp32"),
               dict(workload="yahoo", storage="bf16"),
               dict(workload="yahoo", storage="fp32", schedule="wavefront", workers=888,
                    **{"wf-cols": 15360}, cyclic=True),
               dict(workload="yahoo", storage="fp16", schedule="wavefront", workers=888,
                    **{"wf-cols": 15360}, cyclic=True)],
    "yahoo": [dict(workload="yahoo", storage="fp16"), dict(workload="yahoo", storage="fp32"),
              dict(workload="yahoo", storage="fp32", schedule="wavefront", workers=768),
              dict(workload="yahoo", storage="fp16", schedule="wavefront", workers=768)],
    "wf": [dict(workload="netflix", storage="fp32", schedule="wavefront", workers=768,
                **{"wf-cols": 3072}),
           dict(workload="netflix", storage="fp16", schedule="wavefront", workers=768,
                **{"wf-cols": 3072}),
           dict(workload="netflix", storage="fp32", schedule="wavefront", workers=768,
                **{"wf-cols": 3072}, cyclic=True)],
}


KEYS = ('workers', 'wf-cols', 'cyclic', 'grid-cols', 'group-cols', 'batch-f')


def run(cfg, steps, warmup):
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--steps", str(steps), "--warmup",
           str(warmup), "--no-e2e", "--no-cpu-baseline", "--no-deterministic"]
    for k, v in cfg.items():
        if v is True:
            cmd.append(f"--{k}")
        else:
            cmd += [f"--{k}", str(v)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900)
    try:
        return json.loads(r.stdout.strip().splitlines()[-1])
    except Exception:
        return {"error": (r.stderr or r.stdout)[-300:]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--name", required=True)
    ap.add_argument("--set", default="all")
    ap.add_argument("--steps", type=int, default=8)
    ap.add_argument("--warmup", type=int, default=2)
    a = ap.parse_args()
    cfgs = sum((SETS[s] for s in (SETS if a.set == "all" else a.set.split(","))), [])
    lines = ["| workload | k | storage | schedule | G updates/s | ms/epoch | alg. GB/s | frac of "
             "measured HBM | test RMSE | clocks |", "|---|---|---|---|---|---|---|---|---|---|"]
    rows = []
    for cfg in cfgs:
        d = run(cfg, a.steps, a.warmup)
        rows.append({"cfg": cfg, "result": d})
        if "error" in d:
            lines.append(f"| {cfg} | error: {d['error'][-120:]!r} |")
            continue
        c, rf = d["config"], d["roofline"]
        lines.append(f"| {cfg.get('workload')} {('(' + ', '.join(f'{k}={v}' for k, v in cfg.items() if k in KEYS) + ')') if any(k in cfg for k in KEYS) else ''} | {c['k']} | {c['storage']} | {c['schedule']} | "
                     f"{d['value']/1e9:.3f} | {d['ms_per_step']:.2f} | {rf['step_achieved']:.0f} | "
                     f"{rf['step_frac']:.3f} | {d['test_rmse']:.5f} | {d['clocks']['sm_mhz']} MHz "
                     f"{d['clocks']['reasons']} |")
        print(lines[-1], flush=True)
    out = os.path.join(ROOT, "gpurun_out", a.name + ".md")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")
    with open(out[:-3] + ".json", "w") as f:
        json.dump(rows, f, indent=1)


if __name__ == "__main__":
    main()
