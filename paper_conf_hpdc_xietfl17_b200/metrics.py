"""Per-epoch metrics line (SURVEY 5 "Metrics / logging"): one JSON object per epoch with the
paper's metrics -- #Updates/s (Eq. 7), the "effective memory bandwidth" of the update
stream (algorithmic bytes per second, footnote P:L417) against the HBM peak, test RMSE (Figs. 7b,
9) and the Eq. 2 training loss.  Host logic only: every number comes from the library (CUDA-event
timings, device-counted updates, the RMSE and loss kernels).
"""
from __future__ import annotations

import json
import os
import sys

_ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def hbm_peak_gbs() -> float:
    """MEASURED_PEAKS.json's HBM copy bandwidth when present, else B200_PROFILING.md's fallback."""
    path = os.path.join(_ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            return float(json.load(f)["hbm_gbs"])
    return 6650.0


def epoch_line(ctx, *, test: bool = True, loss: bool = True, hbm_gbs: float | None = None) -> dict:
    """Metrics of the ctx's last epoch (call right after mf_train_epoch)."""
    st = ctx.stats()
    p = ctx.params
    sec = st["epoch_ms"] / 1000.0
    ups = st["updates"] / sec if sec > 0 else 0.0
    gbs = ups * st["bytes_per_update"] / 1e9
    peak = hbm_gbs or hbm_peak_gbs()
    line = {"epoch": ctx.epoch - 1, "mode": {0: "hogwild", 1: "wavefront", 2: "libmf"}[p.schedule],
            "storage": {0: "fp32", 1: "fp16", 2: "bf16"}[p.storage], "k": p.k, "G": max(p.world, 1),
            "m": p.m, "n": p.n, "sec": sec, "sgd_sec": st["sgd_ms"] / 1000.0,
            "updates": st["updates"], "updates_per_s": ups, "alg_GBps": gbs,
            "pct_hbm_roofline": 100.0 * gbs / peak}
    if test:
        line["test_rmse"] = ctx.rmse("test")
    if loss and not p.staged:
        line["train_loss"] = ctx.loss()
    return line


def train(ctx, epochs: int, out=sys.stdout, **kw) -> list[dict]:
    """Run `epochs` epochs, printing one JSON metrics line per epoch to `out`."""
    lines = []
    for _ in range(epochs):
        ctx.train_epoch()
        line = epoch_line(ctx, **kw)
        lines.append(line)
        if out is not None:
            print(json.dumps(line), file=out, flush=True)
    return lines
