"""bench.py -- SGD updates/s of the cuMF_SGD hot path on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl mf|reference]
                    [--workload netflix|yahoo|hugewiki|tiny] [--storage fp16|fp32|bf16]
                    [--schedule hogwild|wavefront] [--k 128] [--emulate-ranks N]

A step is one epoch: the whole hot path (schedule build + SGD kernels [+ strata Q rotation])
over the full synthetic training set, with inputs resident in HBM.  value = updates/s of the
whole job (Eq. 7: epochs x N / elapsed), device-timed with CUDA events on the library stream,
max over ranks.  Prints ONE JSON line on rank 0.

Workloads (BASELINE.json configs): N = 1 runs configs[1] (Netflix-shaped, the metric's
workload); N > 1 runs configs[3] (Hugewiki-shaped DSGD strata, north_star (5)) unless
--workload says otherwise.  For N > 1 launch with torchrun (one rank per GPU, NCCL Q rotation);
--emulate-ranks N runs the same N-rank code path in ONE process on one GPU (ranks are threads,
the library's loopback transport moves the Q segments) -- the CPU-box/1-GPU test of the
multi-rank bench (tests/test_gpu_bench_contract.py).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

HBM_FALLBACK_GBS = 6650.0   # B200_PROFILING.md fallback (only if MEASURED_PEAKS.json is absent)
CPU_SAMPLE = 1 << 23        # oracle sample (ratings) for cpu_baseline
METRIC = "SGD updates/s (Eq. 7: epochs x N / elapsed)"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="mf", choices=["mf", "reference"])
    ap.add_argument("--workload", default=None, choices=["netflix", "yahoo", "hugewiki", "tiny"],
                    help="default: netflix (configs[1]) on 1 GPU; hugewiki (configs[3]) on N > 1")
    ap.add_argument("--storage", default="fp16", choices=["fp16", "fp32", "bf16"])
    ap.add_argument("--schedule", default="hogwild", choices=["hogwild", "wavefront", "libmf"])
    ap.add_argument("--k", type=int, default=128)
    ap.add_argument("--workers", type=int, default=0)
    ap.add_argument("--wf-cols", type=int, default=0)
    ap.add_argument("--cyclic", action="store_true")
    ap.add_argument("--lane-bytes", type=int, default=0)
    ap.add_argument("--prefetch", type=int, default=0)
    ap.add_argument("--wf-kernel", type=int, default=0)
    ap.add_argument("--rating-stage", type=int, default=0,
                    help="Hogwild rating stream: 0 = per-lane loads, 1 = TMA bulk copies")
    ap.add_argument("--group-cols", action="store_true",
                    help="batch-Hogwild with column-grouped batches (reading R24, params.group_cols)")
    ap.add_argument("--plain-batches", action="store_true",
                    help="N > 1: keep the storage order inside batches (no column grouping)")
    ap.add_argument("--exact-order", action="store_true",
                    help="evaluate Alg. 1 l.8-10 in the paper's operation order (params.exact_order)")
    ap.add_argument("--staged", type=int, nargs="?", const=1, default=0,
                    help="out-of-core: 1 = ratings in pinned host memory, streamed per stratum; "
                         "2 = P's row segments too, one strata block at a time")
    ap.add_argument("--grid-a", type=int, default=0)
    ap.add_argument("--grid-cols", type=int, default=0, choices=[0, 1],
                    help="1 = the paper's a x 1 row blocks (P:L379, reading R27), one GPU")
    ap.add_argument("--q-cache", type=int, default=0, choices=[0, 1],
                    help="q_v row loads: 0 = through L1 where the Hogwild kernel has it (reading R28), "
                         "1 = L2 only (params.q_cache)")
    ap.add_argument("--lr-rule", default="eq9", choices=["eq9", "adagrad"])
    ap.add_argument("--batch-f", type=int, default=0, help="Eq. 8 f (0 = 256, P:L277)")
    ap.add_argument("--fraction", type=float, default=1.0, help="scale the workload (testing)")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-deterministic", action="store_true",
                    help="skip the extra deterministic-wavefront line (north_star target run)")
    ap.add_argument("--cpu-sample", type=int, default=CPU_SAMPLE)
    ap.add_argument("--emulate-ranks", type=int, default=0,
                    help="run the N-rank path as N threads on one GPU (loopback transport)")
    return ap.parse_args()


def peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    return HBM_FALLBACK_GBS, "fallback (B200_PROFILING.md)"


def hyper(workload):
    from paper_conf_hpdc_xietfl17_b200 import synth
    if workload == "tiny":
        return dict(lambda_p=0.05, alpha=0.08, beta=0.3, rating_scale=1.0)
    s = synth.SHAPES[workload]
    return dict(lambda_p=s["lam"], alpha=s["alpha"], beta=s["beta"], rating_scale=s["rating_scale"])


def workload(args, device):
    from paper_conf_hpdc_xietfl17_b200 import synth
    if args.workload == "tiny":
        R = synth.tiny(seed=0)
        to = lambda a: torch.from_numpy(a).to(device)  # noqa: E731
        return synth.Ratings(R.m, R.n, to(R.u), to(R.v), to(R.r), to(R.ut), to(R.vt), to(R.rt), R.meta)
    return synth.shaped(args.workload, fraction=args.fraction, device=device)


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index, enabled=True):
        self.dev = device_index
        self.enabled = enabled
        self.p = None
        self.rows = []

    def __enter__(self):
        if not self.enabled:
            return self
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.dev}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except (OSError, FileNotFoundError):
            self.p = None
        return self

    def __exit__(self, *exc):
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
        rows = self.rows
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons, "samples": len(rows)}


# ---------------------------------------------------------------------------------------------
# Rank plumbing: torch.distributed (one process per GPU) or threads of one process (emulation)
# ---------------------------------------------------------------------------------------------
class DistRanks:
    """torch.distributed over NCCL (torchrun): barrier and max/sum over ranks."""

    def __init__(self):
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        self.local = int(os.environ.get("LOCAL_RANK", "0"))
        self.transport = 0
        if self.world > 1:
            import torch.distributed as dist
            torch.cuda.set_device(self.local)
            dist.init_process_group("nccl", device_id=torch.device(f"cuda:{self.local}"))

    def nccl_id(self):
        if self.world == 1:
            return None
        from paper_conf_hpdc_xietfl17_b200 import mf
        return mf.nccl_unique_id_via()

    def barrier(self):
        if self.world > 1:
            import torch.distributed as dist
            dist.barrier()

    def _reduce(self, x, op):
        if self.world == 1:
            return x
        import torch.distributed as dist
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
        return float(t.item())

    def max(self, x):
        return self._reduce(x, "max")

    def sum(self, x):
        return self._reduce(x, "sum")

    def close(self):
        if self.world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


class ThreadGroup:
    """Shared state of N emulated ranks (threads of this process, all on cuda:0)."""

    def __init__(self, world):
        self.world = world
        self.bar = threading.Barrier(world)
        self.slots = [0.0] * world
        self.key = os.urandom(16).ljust(128, b"\0")   # names the library's loopback group


class ThreadRank:
    def __init__(self, group, rank):
        self.g, self.rank, self.world, self.local, self.transport = group, rank, group.world, 0, 1

    def nccl_id(self):
        return self.g.key

    def barrier(self):
        self.g.bar.wait()

    def _reduce(self, x, fn):
        self.g.slots[self.rank] = float(x)
        self.g.bar.wait()
        out = fn(self.g.slots)
        self.g.bar.wait()
        return out

    def max(self, x):
        return self._reduce(x, max)

    def sum(self, x):
        return self._reduce(x, sum)

    def close(self):
        pass


# ---------------------------------------------------------------------------------------------
# Arms
# ---------------------------------------------------------------------------------------------
def cpu_baseline(R, hp, args, sample):
    """The oracle, as it stands, single-threaded on a bounded prefix sample of the workload
    (the training set is drawn iid, so a prefix is a uniform sample); one epoch, timed."""
    from oracle import pyoracle as po
    n = min(sample, R.N)
    u = R.u[:n].cpu().numpy()
    v = R.v[:n].cpu().numpy()
    r = R.r[:n].cpu().numpy()
    m, note = R.m, ""
    if R.m * args.k > (1 << 28):
        # Hugewiki-shaped (m = 50 M): the oracle would initialise a 25.6 GB P for the sample's
        # few rows; compact the sample's row ids to [0, rows present) instead -- the same
        # updates on the same values, in the same order
        rows, u = np.unique(u, return_inverse=True)
        u = u.astype(np.int32)
        m = len(rows)
        note = f"; sample rows compacted to the {m} present"
    o = po.Oracle(m, R.n, args.k, u, v, r, schedule=args.schedule if args.schedule != "libmf"
                  else "hogwild", storage=args.storage,
                  workers=max(1, args.workers) if args.schedule == "wavefront" else 1,
                  wf_cols=args.wf_cols, seed=42, **hp)
    t0 = time.perf_counter()
    o.train_epoch()
    dt = time.perf_counter() - t0
    return {"value": n / dt, "unit": "updates/s", "cores": 1, "kind": "oracle",
            "sample": f"first {n} ratings of the {args.workload}-shaped training set "
                      f"(m={R.m}, n={R.n}, k={args.k}, {args.storage} storage, {args.schedule} "
                      f"serial order), one epoch, single thread; host nproc={os.cpu_count()}"
                      f"{note}",
            "seconds": dt}


def resolve_workload(args, world):
    if args.workload is None:
        args.workload = "netflix" if world == 1 else "hugewiki"
    if world == 1 and args.workload == "hugewiki" and not args.grid_a and not args.grid_cols \
            and args.schedule == "hogwild" and not args.staged:
        # one GPU on the Hugewiki shape: the paper's own blocking, i x j = 64 x 1 (
        # R27).  --grid-a 1 runs the unblocked set.
        args.grid_a, args.grid_cols = 64, 1


def default_f(args, world):
    """Eq. 8 batch f (256).  N > 1 on the Yahoo shape: f = 64 -- each rank's sub-epoch
    launch holds ~1/64 of the ratings, so 256-sample chunks would leave ~1.6 chunks per worker
    and a quantised tail (emulated G = 8: 49.3 -> 54.3 G updates/s, same RMSE;
    profiles/r01_scaling_hot_rows.md section 6).  Column-grouped batches (the N > 1 default on
    the power-law shapes, R24): f = 1024 (profiles/r02_scaling.md)."""
    if args.batch_f:
        return args.batch_f
    if args.group_cols:
        return 1024
    return 64 if (world > 1 and args.workload == "yahoo") else 256


def resolve_group(args, world):
    """N > 1 on the Hugewiki / Netflix shapes: column-grouped batches (R24) by default.  A DSGD
    strata block sees only n/a columns, so a power-law-hot column takes an a-fold larger share
    of its block's updates and Hogwild runs at that column's read-modify-write rate; grouping
    keeps a batch's run of the column in registers.  Emulated Hugewiki (half size) at G = 8:
    10.0 -> 23.4 G updates/s, load imbalance 1.34 -> 1.07 (profiles/r02_scaling.md).
    --plain-batches keeps the paper's storage order inside batches."""
    if world > 1 and args.workload in ("hugewiki", "netflix") and not args.plain_batches \
            and args.schedule == "hogwild":
        args.group_cols = True


def run_reference(args):
    """--impl reference: the CPU oracle on the box's host cores (rank 0 only)."""
    world, rank = int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0"))
    resolve_workload(args, world)
    if rank != 0:
        return
    device = "cuda" if torch.cuda.is_available() else "cpu"
    hp = hyper(args.workload)
    if args.workload == "hugewiki" and args.fraction == 1.0:
        args.fraction = 0.01       # the oracle samples a prefix anyway; 1% keeps generation short
    R = workload(args, device)
    per_step = min(1 << 20, args.cpu_sample)
    vals = []
    for i in range(args.warmup + args.steps):
        cb = cpu_baseline(R, hp, args, per_step)
        if i >= args.warmup:
            vals.append(cb["seconds"])
    n = min(per_step, R.N)
    ms = 1000.0 * float(np.mean(vals))
    value = n / (ms / 1000.0)
    args.gpus = world
    line = {"metric": METRIC, "value": value,
            "unit": "updates/s", "impl": "reference", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": config_of(args, R, world),
            "cpu_baseline": {"value": value, "unit": "updates/s", "cores": 1, "kind": "oracle",
                             "sample": f"each step = one oracle epoch over the first {n} ratings "
                                       f"of the {args.workload}-shaped set"},
            "e2e": {"value": value, "unit": "updates/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def config_of(args, R, world):
    return {"workload": f"{args.workload}-shaped synthetic (Table 2 shape, power-law skew)",
            "m": R.m, "n": R.n, "N_train": R.N, "N_test": R.Ntest, "k": args.k,
            "storage": args.storage, "schedule": args.schedule, "batch_f": default_f(args, world),
            "parallelism": f"dsgd-strata{world}" if world > 1 else "1gpu",
            "fraction": args.fraction, "exact_order": bool(args.exact_order),
            "rating_stage": "tma" if args.rating_stage else "lane-loads",
            "group_cols": bool(args.group_cols),
            "staged": int(args.staged),
            "grid_a": getattr(args, "grid_a_used", None) or args.grid_a or (8 if world > 1 else 1),
            "grid": "a x 1 row blocks" if args.grid_cols == 1 else "a x a strata",
            "q_loads": getattr(args, "q_loads_used", None),
            "l2": "inputs larger than L2 (COO %.2f GB per epoch); model P+Q stays cached as in "
                  "any training run" % (R.N * 12 / 1e9)}


def ncu_traffic(args):
    """DRAM bytes per launch of the SGD kernel from the committed ncu --set full summary of this
    configuration (profiles/ncu_traffic.json), or None."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(path):
        return None, None
    with open(path) as f:
        d = json.load(f)
    a_used = getattr(args, "grid_a_used", None) or args.grid_a or 1
    key = f"{args.workload}/{args.schedule}/{args.storage}/k{args.k}"
    if args.grid_cols:
        key += f"/rows{a_used}"
    if args.schedule == "hogwild" and args.q_cache == 0:
        key += "/qL1"
    e = d.get(key, {})
    # a capture describes one launch configuration: plain or grouped batches of f, full size
    if (e.get("batch_f", 256) != default_f(args, 1) or e.get("group_cols", False) != bool(args.group_cols)
            or e.get("fraction", 1.0) != args.fraction or e.get("grid_cols", 0) != args.grid_cols
            or e.get("grid_a", 1) != a_used or e.get("q_cache", 1) != args.q_cache):
        return None, None
    return e.get("dram_bytes_per_launch"), e.get("source")


def rank_main(args, C, R=None, out=None):
    """Everything one rank does; rank 0 returns (and prints) the JSON line."""
    from paper_conf_hpdc_xietfl17_b200 import mf
    world, rank = C.world, C.rank
    device = torch.device(f"cuda:{C.local}")
    torch.cuda.set_device(device)
    if R is None:
        R = workload(args, device)
    hp = hyper(args.workload)
    big = R.N > (1 << 30)      # Hugewiki-shaped: no second copy of the set for the extra runs
    stream = torch.cuda.Stream(device=device)
    nccl_id = C.nccl_id()
    kw = dict(schedule=args.schedule, storage=args.storage, workers=args.workers,
              wf_cols=args.wf_cols, cyclic=args.cyclic, lane_bytes=args.lane_bytes,
              prefetch=args.prefetch, wf_kernel=args.wf_kernel, grid_a=args.grid_a,
              grid_cols=args.grid_cols, q_cache=args.q_cache,
              batch_f=default_f(args, world), lr_rule=args.lr_rule, seed=42,
              exact_order=args.exact_order, rating_stage=args.rating_stage,
              group_cols=args.group_cols, device=C.local, rank=rank, world=world,
              nccl_id=nccl_id, transport=C.transport, **hp)
    torch.cuda.synchronize()
    model = mf.MF(R.m, R.n, args.k, stream=stream, staged=args.staged, **kw)
    if world > 1:
        print(f"[bench] rank {rank}/{world}: ctx up, transport="
              f"{'nccl' if C.transport == 0 else 'loopback'} (communicator of {world} ranks)",
              file=sys.stderr, flush=True)
    model.load(R.u, R.v, R.r, "train")
    model.load(R.ut, R.vt, R.rt, "test")
    rmse0 = model.rmse("test")
    args.grid_a_used = int(len(model.export("strata", 0)))     # a x 1 with grid_a = 0: auto

    for _ in range(args.warmup):
        model.train_epoch()
    torch.cuda.synchronize()
    if args.schedule == "hogwild" and args.warmup:
        args.q_loads_used = ("L1 (ld.ca; reading R28)" if model.stats()["q_l1"] else "L2 (.cg)")
    C.barrier()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    sgd_ms, sched_ms, updates, launches, sgd_launches = [], [], 0, 0, 0
    st = {}
    with ClockSampler(C.local, enabled=rank == 0) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            model.train_epoch()
            st = model.stats()          # syncs the stream (small gap between epochs, counted)
            sgd_ms.append(st["sgd_ms"])
            sched_ms.append(st["sched_ms"])
            updates += st["updates"]    # counted on the device by the SGD kernels
            launches += st["launches"]
            sgd_launches += st["sgd_launches"]
        ev1.record(stream)
        torch.cuda.synchronize()
    C.barrier()
    ms_total = C.max(ev0.elapsed_time(ev1))
    all_updates = C.sum(float(updates))
    all_launches = C.sum(float(launches))
    visits = model.check_visits()       # exactly-once evidence (after the timed region)
    bad_units = C.sum(float(visits["bad_units"]))
    rmse = model.rmse("test")
    ms_step = ms_total / args.steps
    value = all_updates / (ms_total / 1000.0)
    bpu = st["bytes_per_update"]
    hbm, peak_src = peaks()
    # dominant kernel: the SGD kernel; achieved = algorithmic bytes per launch / avg duration
    per_launch_bytes = updates * bpu / max(sgd_launches, 1)
    avg_launch_ms = float(np.sum(sgd_ms)) / max(sgd_launches, 1)
    achieved = per_launch_bytes / (avg_launch_ms / 1000.0) / 1e9
    traffic, tsrc = ncu_traffic(args) if world == 1 else (None, None)
    roof = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
            "frac": achieved / hbm, "traffic": traffic, "peak_source": peak_src,
            "kernel": f"k_{args.schedule}", "bytes_per_update": bpu, "workers": st["workers"],
            "lanes_per_worker": st["lanes"], "grid": st["grid"],
            "sgd_ms_per_epoch": float(np.mean(sgd_ms)), "sched_ms_per_epoch": float(np.mean(sched_ms)),
            "step_achieved": value / world * bpu / 1e9, "step_frac": value / world * bpu / 1e9 / hbm}
    if traffic:
        # DRAM actually moved per launch (ncu --set full capture of this configuration): the
        # algorithmic fraction above counts the feature rows the L2 serves as HBM bytes
        dram = traffic / (avg_launch_ms / 1000.0) / 1e9
        roof["dram"] = {"achieved": dram, "frac": dram / hbm, "traffic_source": tsrc,
                        "traffic_over_algorithmic": traffic / per_launch_bytes,
                        "limiter": ("a x 1 row blocks: the block's P segment and Q stay in L2, "
                                    "DRAM carries little more than the ratings; L2 latency and the "
                                    "hot q_v rows bound it (profiles/r02_row_blocks.md)")
                                   if args.grid_cols else
                                   ("q_v through L1 (R28): the hot columns are served from L1, the "
                                    "p_u rows stream from DRAM (~220 B per update), and the kernel is "
                                    "bound by memory latency at ~44% issue (profiles/r02_q_l1.md)"
                                    if args.q_cache == 0 and args.workload == "netflix" else
                                    "hot q_v rows (L2 read-modify-write rate of the power-law-hot "
                                    "columns, profiles/r01_scaling_hot_rows.md) on Netflix; DRAM on "
                                    "Yahoo (profiles/r01g_yahoo_fp16_hogwild.md)")}
    model.close()
    del model

    e2e = None
    if not args.no_e2e and not (big and world == 1):
        e2e = run_e2e(args, R, kw, stream, C)
    det = grp = rowb = ql2 = best = None
    if not args.no_deterministic and world == 1 and args.schedule == "hogwild" and not big:
        det = run_deterministic(args, R, hp, stream)
        if not args.group_cols:
            grp = run_variant(args, R, hp, stream, "hogwild, column-grouped batches (R24), f=1024",
                              group_cols=True, batch_f=1024, q_cache=args.q_cache)
        if not args.grid_cols:
            rowb = run_variant(args, R, hp, stream, "hogwild on the a x 1 row-block grid (R27)",
                               grid_cols=1, q_cache=args.q_cache)
        if not args.grid_cols and not args.group_cols:
            best = run_variant(args, R, hp, stream,
                               "hogwild on the a x 1 row-block grid (R27) with column-grouped "
                               "batches (R24), f=1024", grid_cols=1, group_cols=True,
                               batch_f=1024, q_cache=args.q_cache)
        if args.q_cache == 0:
            ql2 = run_variant(args, R, hp, stream, "hogwild, q_v loads through L2 only (q_cache = 1)",
                              q_cache=1, group_cols=bool(args.group_cols),
                              batch_f=default_f(args, world), grid_cols=args.grid_cols)
    cpu = None
    if not args.no_cpu_baseline and rank == 0:
        cpu = cpu_baseline(R, hp, args, args.cpu_sample)
        cpu.pop("seconds", None)
    C.barrier()
    if rank != 0:
        return None
    args.gpus = world
    line = {"metric": METRIC, "value": value,
            "unit": "updates/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "strong" if world > 1 else "weak", "vs_baseline": None,
            "dtype": "f32", "data": "synthetic", "config": config_of(args, R, world),
            "sec_per_epoch": ms_step / 1000.0, "test_rmse": rmse, "test_rmse_init": rmse0,
            "epochs_trained": args.warmup + args.steps,
            "gpu_launches": int(all_launches), "roofline": roof, "clocks": clk.summary(),
            "exactly_once": {"bad_units": int(bad_units), "units": visits["units"],
                             "epochs": visits["epochs"], "updates_per_epoch": all_updates / args.steps,
                             "N": R.N},
            "e2e": e2e, "cpu_baseline": cpu, "deterministic": det, "grouped": grp,
            "row_blocks": rowb, "row_blocks_grouped": best, "q_l2_only": ql2,
            "paper_context": "cuMF_SGD Table 5 (P:L414-415), fp16 Hogwild: Netflix 267M/s TITAN X, "
                             "613M/s P100; Hugewiki 256M/s / 710M/s (other hardware; context only)"}
    if isinstance(C, ThreadRank):
        line["emulated_ranks"] = {"ranks": world, "transport": "loopback (one process, one GPU)",
                                  "note": "code-path test of the N-rank bench: all ranks share "
                                          "cuda:0, so the numbers are not a scaling result"}
    if out is not None:
        out.append(line)
    return line


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


def run_variant(args, R, hp, stream, label, **variant):
    """The same Hogwild run in another of the method's configurations, device-timed like the
    main line, on the same data: `grouped` = column-grouped batches (reading R24,
    params.group_cols) at f = 1024 (profiles/r02_grouped_batches.md); `row_blocks` = the paper's
    a x 1 row-block grid (reading R27; params.grid_cols = 1, a picked so that a P row
    segment is ~32 MiB: profiles/r02_row_blocks.md)."""
    from paper_conf_hpdc_xietfl17_b200 import mf
    steps, warm = max(3, args.steps // 2), 3
    m = mf.MF(R.m, R.n, args.k, stream=stream, schedule="hogwild", storage=args.storage,
              seed=42, **hp, **variant)
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
    out = {"schedule": label, "storage": args.storage,
           "value": upd / (ms / 1000.0), "unit": "updates/s", "ms_per_step": ms / steps,
           "steps": steps, "warmup": warm, "test_rmse": m.rmse("test"),
           "exactly_once_bad_units": m.check_visits()["bad_units"],
           "sgd_launches_per_epoch": st["sgd_launches"],
           "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                        "frac": achieved / hbm, "bytes_per_update": bpu}}
    if variant.get("grid_cols"):
        out["grid_a"] = int(len(m.export("strata", 0)))
    m.close()
    return out


def run_e2e(args, R, kw, stream, C):
    """The same metric through the public API with the ratings in HOST memory: a ctx in the
    paper's out-of-core mode (staged = 1, section 6.2) keeps the rank's bucketed
    ratings in pinned host memory and copies each epoch's ratings host -> device (cudaMemcpyAsync
    on a copy stream, overlapped with the previous stratum's compute); every step is one epoch
    plus the test RMSE read back to the host (D2H).  Host wall clock around K synchronised steps
    (max over ranks), after the one-time load and a warm-up epoch.  At N = 1 the ctx loads the
    caller's COO from pinned host memory, and the cold path (mf_create + mf_load_coo from pinned
    host + 1 epoch + mf_rmse) is reported too; at N > 1 every rank loads the (device-resident)
    full set and keeps its own row segments, as in the resident run."""
    from paper_conf_hpdc_xietfl17_b200 import mf
    world = C.world
    kw2 = dict(kw)
    kw2["staged"] = max(1, int(args.staged))
    host = None
    if world == 1:
        host = [x.cpu().pin_memory().numpy() for x in (R.u, R.v, R.r, R.ut, R.vt, R.rt)]
    m = mf.MF(R.m, R.n, args.k, stream=stream, **kw2)
    if host is not None:
        m.load(host[0], host[1], host[2], "train", on_device=False)
        m.load(host[3], host[4], host[5], "test", on_device=False)
    else:
        m.load(R.u, R.v, R.r, "train")
        m.load(R.ut, R.vt, R.rt, "test")
    m.train_epoch()
    m.rmse("test")
    steps = max(3, args.e2e_steps * 2)
    torch.cuda.synchronize()
    C.barrier()
    t0 = time.perf_counter()
    for _ in range(steps):
        m.train_epoch()
        m.rmse("test")                 # synchronises; 8-byte D2H
    dt = C.max((time.perf_counter() - t0) / steps)
    h2d = int(C.sum(float(m.stats()["h2d_bytes"])))   # the last epoch's H2D over all ranks
    m.close()
    out = {"value": R.N / dt, "unit": "updates/s", "ms_per_step": 1000 * dt, "steps": steps,
           "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": 8 * world,
           "what": "per step: mf_train_epoch in out-of-core mode (staged=1: the epoch's ratings "
                   "copied from pinned host memory, packed to 9-10 B per rating, "
                   "overlapped with compute) + mf_rmse (D2H); host wall clock, max over ranks"}
    if world > 1:
        return out
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
    out["cold"] = {"value": R.N / dc, "unit": "updates/s", "ms_per_step": 1000 * dc,
                   "h2d_bytes_per_step": int(12 * (R.N + R.Ntest)), "d2h_bytes_per_step": 8,
                   "what": "per step: mf_create + mf_load_coo(train,test from pinned host; the "
                           "whole one-time GPU preprocessing) + 1 epoch + mf_rmse"}
    return out


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    if args.emulate_ranks > 1:
        world = args.emulate_ranks
        resolve_workload(args, world)
        resolve_group(args, world)
        torch.cuda.set_device(0)
        R = workload(args, torch.device("cuda:0"))
        group = ThreadGroup(world)
        out, errs = [], []

        def work(rank):
            try:
                rank_main(args, ThreadRank(group, rank), R, out)
            except BaseException as e:  # noqa: BLE001 -- surface in the main thread
                errs.append(e)
                group.bar.abort()

        th = [threading.Thread(target=work, args=(r,)) for r in range(world)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        if errs:
            raise errs[0]
        print(json.dumps(out[0]), flush=True)
        return
    C = DistRanks()
    resolve_workload(args, C.world)
    resolve_group(args, C.world)
    line = rank_main(args, C)
    if line is not None:
        print(json.dumps(line), flush=True)
    C.close()


if __name__ == "__main__":
    main()
