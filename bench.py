"""bench.py -- SGD updates/s of the cuMF_SGD hot path on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl mf|reference]
                    [--workload netflix|yahoo|hugewiki|tiny] [--storage fp16|fp32|bf16]
                    [--schedule hogwild|wavefront] [--k 128]

A step is one epoch: the whole hot path (schedule build + SGD kernels [+ strata Q rotation])
over the full synthetic training set, with inputs resident in HBM.  value = updates/s of the
whole job (Eq. 7: epochs x N / elapsed), device-timed with CUDA events on the library stream,
max over ranks.  Prints ONE JSON line on rank 0.  For N > 1 launch with torchrun (one rank per
GPU); the ranks run DSGD strata with NCCL Q rotation.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

HBM_FALLBACK_GBS = 6650.0   # B200_PROFILING.md fallback (only if MEASURED_PEAKS.json is absent)
CPU_SAMPLE = 1 << 23        # oracle sample (ratings) for cpu_baseline


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="mf", choices=["mf", "reference"])
    ap.add_argument("--workload", default=None, choices=["netflix", "yahoo", "hugewiki", "tiny"],
                    help="default: netflix (configs[1]) on 1 GPU; yahoo (configs[2]) on N > 1 "
                         "(DESIGN.md section 8: the set DSGD strata scale on)")
    ap.add_argument("--storage", default="fp16", choices=["fp16", "fp32", "bf16"])
    ap.add_argument("--schedule", default="hogwild", choices=["hogwild", "wavefront", "libmf"])
    ap.add_argument("--k", type=int, default=128)
    ap.add_argument("--workers", type=int, default=0)
    ap.add_argument("--wf-cols", type=int, default=0)
    ap.add_argument("--cyclic", action="store_true")
    ap.add_argument("--lane-bytes", type=int, default=0)
    ap.add_argument("--prefetch", type=int, default=0)
    ap.add_argument("--wf-kernel", type=int, default=0)
    ap.add_argument("--staged", action="store_true",
                    help="out-of-core: ratings in pinned host memory, streamed per stratum")
    ap.add_argument("--grid-a", type=int, default=0)
    ap.add_argument("--lr-rule", default="eq9", choices=["eq9", "adagrad"])
    ap.add_argument("--batch-f", type=int, default=0, help="Eq. 8 f (0 = 256, P:L277)")
    ap.add_argument("--fraction", type=float, default=1.0, help="scale the workload (testing)")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-deterministic", action="store_true",
                    help="skip the extra deterministic-wavefront line (north_star target run)")
    ap.add_argument("--cpu-sample", type=int, default=CPU_SAMPLE)
    return ap.parse_args()


def peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    return HBM_FALLBACK_GBS, "fallback (B200_PROFILING.md)"


def workload(args, device):
    from paper_conf_hpdc_xietfl17_b200 import synth
    if args.workload == "tiny":
        R = synth.tiny(seed=0)
        hp = dict(lambda_p=0.05, alpha=0.08, beta=0.3, rating_scale=1.0)
        to = lambda a: torch.from_numpy(a).to(device)  # noqa: E731
        R = synth.Ratings(R.m, R.n, to(R.u), to(R.v), to(R.r), to(R.ut), to(R.vt), to(R.rt), R.meta)
        return R, hp
    s = synth.SHAPES[args.workload]
    R = synth.shaped(args.workload, fraction=args.fraction, device=device)
    hp = dict(lambda_p=s["lam"], alpha=s["alpha"], beta=s["beta"], rating_scale=s["rating_scale"])
    return R, hp


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index):
        self.dev = device_index
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.dev}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except (OSError, FileNotFoundError):
            self.p = None
        return self

    def __exit__(self, *exc):
        self.rows = []
        if self.p is None:
            return
        time.sleep(0.25)
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) >= 9:
                self.rows.append(f)

    def summary(self):
        rows = getattr(self, "rows", [])
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons, "samples": len(rows)}


def dist_setup(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
    return world, rank, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(x, world):
    if world == 1:
        return x
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x, world):
    if world == 1:
        return x
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t)
    return float(t.item())


def cpu_baseline(R, hp, args, sample):
    """The oracle, as it stands, single-threaded on a bounded prefix sample of the workload
    (the training set is drawn iid, so a prefix is a uniform sample); one epoch, timed."""
    from oracle import pyoracle as po
    n = min(sample, R.N)
    u = R.u[:n].cpu().numpy()
    v = R.v[:n].cpu().numpy()
    r = R.r[:n].cpu().numpy()
    o = po.Oracle(R.m, R.n, args.k, u, v, r, schedule=args.schedule, storage=args.storage,
                  workers=max(1, args.workers) if args.schedule == "wavefront" else 1,
                  wf_cols=args.wf_cols, seed=42, **hp)
    t0 = time.perf_counter()
    o.train_epoch()
    dt = time.perf_counter() - t0
    return {"value": n / dt, "unit": "updates/s", "cores": 1, "kind": "oracle",
            "sample": f"first {n} ratings of the {args.workload}-shaped training set "
                      f"(m={R.m}, n={R.n}, k={args.k}, {args.storage} storage, {args.schedule} "
                      f"serial order), one epoch, single thread; host nproc={os.cpu_count()}",
            "seconds": dt}


def resolve_workload(args, world):
    if args.workload is None:
        args.workload = "netflix" if world == 1 else "yahoo"


def run_reference(args):
    """--impl reference: the CPU oracle on the box's host cores (rank 0 only)."""
    world, rank, local = int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")), 0
    resolve_workload(args, world)
    if rank != 0:
        return
    device = "cuda" if torch.cuda.is_available() else "cpu"
    R, hp = workload(args, device)
    per_step = min(1 << 20, args.cpu_sample)
    vals = []
    for i in range(args.warmup + args.steps):
        cb = cpu_baseline(R, hp, args, per_step)
        if i >= args.warmup:
            vals.append(cb["seconds"])
    n = min(per_step, R.N)
    ms = 1000.0 * float(np.mean(vals))
    value = n / (ms / 1000.0)
    line = {"metric": "SGD updates/s (Eq. 7: epochs x N / elapsed)", "value": value,
            "unit": "updates/s", "impl": "reference", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": config_of(args, R),
            "cpu_baseline": {"value": value, "unit": "updates/s", "cores": 1, "kind": "oracle",
                             "sample": f"each step = one oracle epoch over the first {n} ratings"},
            "e2e": {"value": value, "unit": "updates/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def config_of(args, R):
    return {"workload": f"{args.workload}-shaped synthetic (Table 2 shape, power-law skew)",
            "m": R.m, "n": R.n, "N_train": R.N, "N_test": R.Ntest, "k": args.k,
            "storage": args.storage, "schedule": args.schedule,
            "batch_f": args.batch_f or (64 if args.gpus > 1 else 256),
            "parallelism": f"dsgd-strata{args.gpus}" if args.gpus > 1 else "1gpu",
            "staged": bool(args.staged), "grid_a": args.grid_a or (8 if args.gpus > 1 else 1),
            "l2": "inputs larger than L2 (COO %.2f GB per epoch); model P+Q stays cached as in "
                  "any training run" % (R.N * 12 / 1e9)}


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    world, rank, local = dist_setup(args)
    args.gpus = world
    resolve_workload(args, world)
    device = torch.device(f"cuda:{local}")
    torch.cuda.set_device(device)
    from paper_conf_hpdc_xietfl17_b200 import mf

    R, hp = workload(args, device)
    if R.N > (1 << 30):       # Hugewiki-shaped: no second copy of the set for e2e / extra runs
        args.no_e2e = args.no_cpu_baseline = args.no_deterministic = True
    stream = torch.cuda.Stream(device=device)
    nccl_id = None
    if world > 1:
        nccl_id = mf.nccl_unique_id_via()
    kw = dict(schedule=args.schedule, storage=args.storage, workers=args.workers,
              wf_cols=args.wf_cols, cyclic=args.cyclic, lane_bytes=args.lane_bytes, prefetch=args.prefetch,
              wf_kernel=args.wf_kernel, staged=args.staged, grid_a=args.grid_a,
              # N > 1: f = 64.  Each rank's sub-epoch launch holds ~1/64 of the ratings, so
              # 256-sample chunks leave ~1.6 chunks per worker and a quantised tail; emulated on
              # Yahoo at G = 8: 49.3 (f = 256) -> 54.3 G updates/s (f = 64), same RMSE
              # (profiles/r01_scaling_hot_rows.md section 6; f is Eq. 8's free batch)
              batch_f=args.batch_f or (64 if world > 1 else 256),
              lr_rule=args.lr_rule, seed=42,
              device=local, rank=rank, world=world, nccl_id=nccl_id, **hp)
    torch.cuda.synchronize()
    model = mf.MF(R.m, R.n, args.k, stream=stream, **kw)
    model.load(R.u, R.v, R.r, "train")
    model.load(R.ut, R.vt, R.rt, "test")
    rmse0 = model.rmse("test")

    for _ in range(args.warmup):
        model.train_epoch()
    torch.cuda.synchronize()
    barrier(world)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    sgd_ms, sched_ms, updates, launches, sgd_launches = [], [], 0, 0, 0
    st = {}
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            model.train_epoch()
            st = model.stats()          # syncs the stream (small gap between epochs, counted)
            sgd_ms.append(st["sgd_ms"])
            sched_ms.append(st["sched_ms"])
            updates += st["updates"]
            launches += st["launches"]
            sgd_launches += st["sgd_launches"]
        ev1.record(stream)
        torch.cuda.synchronize()
    barrier(world)
    ms_total = max_over_ranks(ev0.elapsed_time(ev1), world)
    all_updates = sum_over_ranks(float(updates), world)
    rmse = model.rmse("test")
    ms_step = ms_total / args.steps
    value = all_updates / (ms_total / 1000.0)
    bpu = st["bytes_per_update"]
    hbm, peak_src = peaks()
    # dominant kernel: the SGD kernel; achieved = algorithmic bytes per launch / avg duration
    per_launch_bytes = updates * bpu / max(sgd_launches, 1)
    avg_launch_ms = float(np.sum(sgd_ms)) / max(sgd_launches, 1)
    achieved = per_launch_bytes / (avg_launch_ms / 1000.0) / 1e9
    traffic = ncu_traffic(args)
    roof = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
            "frac": achieved / hbm, "traffic": traffic, "peak_source": peak_src,
            "kernel": f"k_{args.schedule}", "bytes_per_update": bpu,
            "sgd_ms_per_epoch": float(np.mean(sgd_ms)), "sched_ms_per_epoch": float(np.mean(sched_ms)),
            "step_achieved": value / world * bpu / 1e9, "step_frac": value / world * bpu / 1e9 / hbm}
    model.close()
    del model

    e2e = None
    if not args.no_e2e and world == 1:
        e2e = run_e2e(args, R, kw, stream)
    det = None
    if not args.no_deterministic and world == 1 and args.schedule == "hogwild":
        det = run_deterministic(args, R, hp, stream)
    cpu = None
    if not args.no_cpu_baseline and world == 1 and rank == 0:
        cpu = cpu_baseline(R, hp, args, args.cpu_sample)
        cpu.pop("seconds", None)
    if rank == 0:
        line = {"metric": "SGD updates/s (Eq. 7: epochs x N / elapsed)", "value": value,
                "unit": "updates/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": ms_step, "higher_is_better": True,
                "scaling": "strong" if world > 1 else "weak", "vs_baseline": None,
                "dtype": "f32", "data": "synthetic", "config": config_of(args, R),
                "sec_per_epoch": ms_step / 1000.0, "test_rmse": rmse, "test_rmse_init": rmse0,
                "epochs_trained": args.warmup + args.steps,
                "gpu_launches": int(launches), "roofline": roof, "clocks": clk.summary(),
                "e2e": e2e, "cpu_baseline": cpu, "deterministic": det,
                "paper_context": "cuMF_SGD Table 5 (P:L414-415), Netflix fp16 Hogwild: 267M/s "
                                 "TITAN X, 613M/s P100 (other hardware; context only)"}
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


def run_deterministic(args, R, hp, stream):
    """The north_star target run: the deterministic conflict-free wavefront (oracle-exact
    order), fp32 storage, k = args.k, s = 888 workers (all co-resident: 6 per SM at 32 KB of
    ring each), cyclic column order with c = 7680 (SURVEY App. A cyclic variant; s and c from
    the sweep in profiles/r01_wavefront_sweep.md), on the same data; device-timed like the main
    line."""
    from paper_conf_hpdc_xietfl17_b200 import mf
    steps, warm = max(3, args.steps // 2), 2
    s_w = min(888, max(1, R.m // 4))                  # (clamped only for --fraction test runs)
    c_w = max(s_w, min(7680, R.n))
    m = mf.MF(R.m, R.n, args.k, stream=stream, schedule="wavefront", storage="fp32", workers=s_w,
              wf_cols=c_w, cyclic=True, seed=42, **hp)
    m.load(R.u, R.v, R.r, "train")
    m.load(R.ut, R.vt, R.rt, "test")
    for _ in range(warm):
        m.train_epoch()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    sgd, upd = [], 0
    e0.record(stream)
    for _ in range(steps):
        m.train_epoch()
        st = m.stats()
        sgd.append(st["sgd_ms"])
        upd += st["updates"]
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    hbm, _ = peaks()
    bpu = st["bytes_per_update"]
    achieved = upd * bpu / (float(np.sum(sgd)) / 1000.0) / 1e9
    out = {"schedule": f"wavefront (deterministic, cyclic, s={s_w}, c={c_w})", "storage": "fp32",
           "value": upd / (ms / 1000.0), "unit": "updates/s", "ms_per_step": ms / steps,
           "steps": steps, "warmup": warm, "test_rmse": m.rmse("test"),
           "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                        "frac": achieved / hbm, "bytes_per_update": bpu,
                        "step_frac": upd / (ms / 1000.0) * bpu / 1e9 / hbm}}
    m.close()
    return out


def run_e2e(args, R, kw, stream):
    """The same metric through the public API with the ratings in HOST memory: a ctx in the
    paper's out-of-core mode (staged = 1, section 6.2) keeps the bucketed ratings
    in pinned host memory and copies each epoch's ratings host -> device (cudaMemcpyAsync on a
    copy stream, overlapped with the previous epoch's compute); every step is one epoch plus the
    test RMSE read back to the host (D2H).  Host wall clock around K synchronised steps, after
    the one-time load and a warm-up epoch.  Also reported: the cold path (mf_create + mf_load_coo
    from pinned host + 1 epoch + mf_rmse per step), which includes the one-time preprocessing."""
    from paper_conf_hpdc_xietfl17_b200 import mf
    host = [x.cpu().pin_memory().numpy() for x in (R.u, R.v, R.r, R.ut, R.vt, R.rt)]
    kw2 = dict(kw)
    kw2["staged"] = True
    m = mf.MF(R.m, R.n, args.k, stream=stream, **kw2)
    m.load(host[0], host[1], host[2], "train", on_device=False)
    m.load(host[3], host[4], host[5], "test", on_device=False)
    m.train_epoch()
    m.rmse("test")
    steps = max(3, args.e2e_steps * 2)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(steps):
        m.train_epoch()
        m.rmse("test")                 # synchronises; 8-byte D2H
    dt = (time.perf_counter() - t0) / steps
    h2d = int(m.stats()["h2d_bytes"])    # the last epoch's H2D (packed 10 B/rating when n < 2^16)
    m.close()
    cold = []
    for i in range(args.e2e_steps + 1):
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        c = mf.MF(R.m, R.n, args.k, stream=stream, **kw)
        c.load(host[0], host[1], host[2], "train", on_device=False)
        c.load(host[3], host[4], host[5], "test", on_device=False)
        c.train_epoch()
        c.rmse("test")
        torch.cuda.synchronize()
        if i > 0:           # first iteration warms the allocator / module load
            cold.append(time.perf_counter() - t1)
        c.close()
    dc = float(np.mean(cold))
    return {"value": R.N / dt, "unit": "updates/s", "ms_per_step": 1000 * dt, "steps": steps,
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": 8,
            "what": "per step: mf_train_epoch in out-of-core mode (staged=1: the epoch's ratings "
                    "copied from pinned host memory, packed to 10 B per rating, overlapped with "
                    "compute) + mf_rmse (D2H); host wall clock",
            "cold": {"value": R.N / dc, "unit": "updates/s", "ms_per_step": 1000 * dc,
                     "h2d_bytes_per_step": int(12 * (R.N + R.Ntest)), "d2h_bytes_per_step": 8,
                     "what": "per step: mf_create + mf_load_coo(train,test from pinned host; the "
                             "whole one-time GPU preprocessing) + 1 epoch + mf_rmse"}}


def ncu_traffic(args):
    """DRAM bytes per launch of the SGD kernel from the committed ncu --set full summary of this
    configuration (profiles/), or None."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(path):
        return None
    with open(path) as f:
        d = json.load(f)
    key = f"{args.workload}/{args.schedule}/{args.storage}/k{args.k}"
    return d.get(key, {}).get("dram_bytes_per_launch")


if __name__ == "__main__":
    main()
