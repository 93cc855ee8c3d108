"""ctypes binding of libmf_b200.so (include/mf.h): argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels.  There is no CPU fallback:
if the library is missing or the device is unavailable, the calls raise.  PyTorch is used for
device memory (the optional caching-allocator hooks), streams (``torch.cuda.current_stream``)
and, in the multi-GPU mode, the process group that broadcasts the ncclUniqueId.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("MF_LIB", os.path.join(HERE, "libmf_b200.so"))   # MF_LIB: a variant build (tools/)

STORAGE = {"fp32": 0, "fp16": 1, "bf16": 2}
SCHEDULE = {"hogwild": 0, "wavefront": 1, "libmf": 2}
SETS = {"train": 0, "test": 1}
EXPORTS = {"perm": 0, "rho_r": 1, "rho_c": 2, "blockid": 3, "chunkorder": 4, "wfseq": 5,
           "tickets": 6, "strata": 7}
STATUS = {0: "MF_OK", -1: "MF_E_INVAL", -2: "MF_E_NOMEM", -3: "MF_E_CUDA", -4: "MF_E_NCCL",
          -5: "MF_E_STATE", -6: "MF_E_RANGE", -7: "MF_E_UNSUPPORTED"}


class MFError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)


class Allocator(ctypes.Structure):
    _fields_ = [("alloc", _ALLOC_FN), ("free", _FREE_FN), ("user", ctypes.c_void_p)]


class Params(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_uint32), ("m", ctypes.c_int64), ("n", ctypes.c_int64),
                ("k", ctypes.c_int32), ("lambda_p", ctypes.c_float), ("lambda_q", ctypes.c_float),
                ("alpha", ctypes.c_float), ("beta", ctypes.c_float),
                ("init_scale", ctypes.c_float), ("rating_scale", ctypes.c_float),
                ("seed", ctypes.c_uint64), ("schedule", ctypes.c_int32),
                ("storage", ctypes.c_int32), ("workers", ctypes.c_int32),
                ("batch_f", ctypes.c_int32), ("wf_cols", ctypes.c_int32),
                ("grid_a", ctypes.c_int32), ("cyclic", ctypes.c_int32),
                ("lane_bytes", ctypes.c_int32), ("prefetch", ctypes.c_int32),
                ("lr_rule", ctypes.c_int32), ("ada_eps", ctypes.c_float),
                ("staged", ctypes.c_int32), ("wf_kernel", ctypes.c_int32),
                ("device", ctypes.c_int32),
                ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("transport", ctypes.c_int32), ("nccl_id", ctypes.c_void_p),
                ("stream", ctypes.c_void_p), ("alloc", ctypes.POINTER(Allocator)),
                ("launch_blocks", ctypes.c_int32), ("exact_order", ctypes.c_int32),
                ("rating_stage", ctypes.c_int32), ("stage_chunk", ctypes.c_int64),
                ("group_cols", ctypes.c_int32), ("check_owners", ctypes.c_int32),
                ("grid_cols", ctypes.c_int32), ("q_cache", ctypes.c_int32)]


class Stats(ctypes.Structure):
    _fields_ = [("epoch_ms", ctypes.c_double), ("sgd_ms", ctypes.c_double),
                ("sched_ms", ctypes.c_double), ("comm_ms", ctypes.c_double),
                ("sgd_launches", ctypes.c_int64), ("launches", ctypes.c_int64),
                ("updates", ctypes.c_int64), ("bytes_per_update", ctypes.c_int64),
                ("workers", ctypes.c_int32), ("lanes", ctypes.c_int32),
                ("grid", ctypes.c_int32), ("block", ctypes.c_int32), ("h2d_bytes", ctypes.c_int64),
                ("q_l1", ctypes.c_int32)]


_lib = None
EXPORTED = ["mf_abi_version", "mf_params_default", "mf_create", "mf_load_coo", "mf_train_epoch",
            "mf_rmse", "mf_loss", "mf_get_factors", "mf_set_factors", "mf_set_epoch", "mf_get_epoch",
            "mf_export_schedule", "mf_get_stats", "mf_get_launch_ms", "mf_check_visits",
            "mf_owner_violations",
            "mf_strata_holders", "mf_strata_plan", "mf_comm_selftest",
            "mf_destroy",
            "mf_last_error", "mf_status_string"]


def lib() -> ctypes.CDLL:
    """Load libmf_b200.so (raises if it has not been built: no fallback path exists)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is not built; run `python -m paper_conf_hpdc_xietfl17_b200.build`"
                          " (the CUDA path has no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    i32, i64, u64, vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_void_p
    sig = {
        "mf_abi_version": (i32, []),
        "mf_params_default": (i32, [ctypes.POINTER(Params)]),
        "mf_create": (i32, [ctypes.POINTER(Params), ctypes.POINTER(vp)]),
        "mf_load_coo": (i32, [vp, i32, i64, vp, vp, vp, i32]),
        "mf_train_epoch": (i32, [vp, ctypes.POINTER(i32)]),
        "mf_rmse": (i32, [vp, i32, ctypes.POINTER(ctypes.c_double)]),
        "mf_loss": (i32, [vp, ctypes.POINTER(ctypes.c_double)]),
        "mf_get_factors": (i32, [vp, vp, vp, i32]),
        "mf_set_factors": (i32, [vp, vp, vp, i32]),
        "mf_set_epoch": (i32, [vp, i32]),
        "mf_get_epoch": (i32, [vp, ctypes.POINTER(i32)]),
        "mf_export_schedule": (i32, [vp, i32, i32, vp, ctypes.POINTER(i64)]),
        "mf_get_stats": (i32, [vp, ctypes.POINTER(Stats)]),
        "mf_get_launch_ms": (i32, [vp, vp, ctypes.POINTER(i64)]),
        "mf_check_visits": (i32, [vp, ctypes.POINTER(i64), ctypes.POINTER(i64), ctypes.POINTER(i32)]),
        "mf_owner_violations": (i32, [vp, ctypes.POINTER(i64)]),
        "mf_strata_holders": (i32, [u64, i32, i32, i32, i32, vp]),
        "mf_strata_plan": (i32, [u64, i32, i32, i32, i64, i32, i32, vp, vp, vp, vp, vp]),
        "mf_comm_selftest": (i32, [vp, i32, i32, i32, i32, ctypes.c_char_p, i32]),
        "mf_destroy": (None, [vp]),
        "mf_last_error": (ctypes.c_char_p, [vp]),
        "mf_status_string": (ctypes.c_char_p, [i32]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    _lib = L
    return L


def strata_holders(seed: int, a: int, world: int, t: int, j: int) -> list[int]:
    """Host-only planner: rank holding each Q segment in sub-epoch j of epoch t."""
    out = (ctypes.c_int32 * a)()
    st = lib().mf_strata_holders(seed, a, world, t, j, out)
    if st != 0:
        raise MFError(st, "mf_strata_holders")
    return list(out)


def strata_plan(seed: int, a: int, world: int, rank: int, n: int, t: int, j: int, holders):
    """Host-only plan of sub-epoch j (the one mf_train_epoch executes): returns
    (blocks, transfers, new_holders); transfers = [(J, src, dst, lo, hi), ...]."""
    h = (ctypes.c_int32 * a)(*holders)
    blocks = (ctypes.c_int64 * a)()
    xf = (ctypes.c_int64 * (5 * a))()
    nb, nx = ctypes.c_int32(0), ctypes.c_int32(0)
    st = lib().mf_strata_plan(seed, a, world, rank, n, t, j, h, blocks, ctypes.byref(nb), xf,
                              ctypes.byref(nx))
    if st != 0:
        raise MFError(st, "mf_strata_plan")
    tr = [tuple(xf[5 * i:5 * i + 5]) for i in range(nx.value)]
    return list(blocks[:nb.value]), tr, list(h)


def comm_selftest(comm_id: bytes, world: int = 1, rank: int = 0, device: int = 0,
                  transport: int = 0) -> str:
    """Run the strata transport's primitives (all-reduce, broadcast, rotation-shaped send/recv,
    segment gather) on `device` and check them (mf_comm_selftest); returns the report line,
    raises MFError on a failed call or a wrong value."""
    idb = ctypes.create_string_buffer(bytes(comm_id).ljust(128, b"\0")[:128], 128)
    out = ctypes.create_string_buffer(256)
    st = lib().mf_comm_selftest(ctypes.cast(idb, ctypes.c_void_p), world, rank, device, transport,
                                out, 256)
    if st != 0:
        raise MFError(st, "mf_comm_selftest: " + out.value.decode(errors="replace"))
    return out.value.decode()


def _torch():
    import torch
    return torch


class _TorchAllocator:
    """mf_allocator hooks backed by torch's CUDA caching allocator.  `budget` (bytes, optional)
    caps the ctx's live device memory: an allocation beyond it returns NULL (MF_E_NOMEM), the
    way a device smaller than the problem would; `peak` records the high-water mark."""

    def __init__(self, device: int, budget: int | None = None):
        torch = _torch()
        self.device = device
        self.budget = budget              # may be raised between a failed and a retried load
        self.sizes = {}
        self.live = 0
        self.peak = 0

        def _alloc(nbytes, stream, user):
            if self.budget is not None and self.live + int(nbytes) > self.budget:
                return None
            try:
                ptr = torch.cuda.caching_allocator_alloc(int(nbytes), device, int(stream or 0))
            except Exception:  # OOM -> NULL -> MF_E_NOMEM
                return None
            self.sizes[ptr] = int(nbytes)
            self.live += int(nbytes)
            self.peak = max(self.peak, self.live)
            return ptr

        def _free(ptr, nbytes, stream, user):
            if ptr:
                self.live -= self.sizes.pop(ptr, 0)
                torch.cuda.caching_allocator_delete(ptr)

        self._a = _ALLOC_FN(_alloc)
        self._f = _FREE_FN(_free)
        self.struct = Allocator(self._a, self._f, None)


def _as_ptr(x, dtype, on_device: bool):
    """(pointer, keepalive) for a numpy array or torch tensor of the given dtype."""
    if on_device:
        torch = _torch()
        t = x if isinstance(x, torch.Tensor) else torch.as_tensor(x)
        want = {np.int32: torch.int32, np.float32: torch.float32}[dtype]
        t = t.to(dtype=want).contiguous()
        return ctypes.c_void_p(t.data_ptr()), t
    a = np.ascontiguousarray(x, dtype=dtype)
    return ctypes.c_void_p(a.ctypes.data), a


class MF:
    """One training context (one GPU / one rank).  Mirrors include/mf.h."""

    def __init__(self, m: int, n: int, k: int = 128, *, lambda_p: float = 0.05,
                 lambda_q: float | None = None, alpha: float = 0.08, beta: float = 0.3,
                 init_scale: float = 1.0, rating_scale: float = 1.0, seed: int = 42,
                 schedule: str = "hogwild", storage: str = "fp32", workers: int = 0,
                 batch_f: int = 256, wf_cols: int = 0, grid_a: int = 0, cyclic: bool = False,
                 lane_bytes: int = 0, prefetch: int = 0, wf_kernel: int = 0, staged: bool = False,
                 lr_rule: str = "eq9", ada_eps: float = 1e-8, launch_blocks: int = 0,
                 exact_order: bool = False, rating_stage: int = 0, stage_chunk: int = 0,
                 group_cols: bool = False, check_owners: bool = False, grid_cols: int = 0,
                 q_cache: int = 0, device: int = 0, rank: int = 0, world: int = 1,
                 nccl_id: bytes | None = None, transport: int = 0, stream=None,
                 allocator: str = "torch", device_budget: int | None = None):
        L = lib()
        p = Params()
        L.mf_params_default(ctypes.byref(p))
        p.m, p.n, p.k = int(m), int(n), int(k)
        p.lambda_p = lambda_p
        p.lambda_q = lambda_p if lambda_q is None else lambda_q
        p.alpha, p.beta, p.init_scale, p.rating_scale = alpha, beta, init_scale, rating_scale
        p.seed = seed
        p.schedule, p.storage = SCHEDULE[schedule], STORAGE[storage]
        p.workers, p.batch_f, p.wf_cols, p.grid_a = workers, batch_f, wf_cols, grid_a
        p.cyclic, p.lane_bytes, p.prefetch, p.wf_kernel = int(cyclic), lane_bytes, prefetch, wf_kernel
        p.staged = int(staged)
        p.launch_blocks = launch_blocks
        p.exact_order = int(exact_order)
        p.rating_stage = int(rating_stage)
        p.stage_chunk = int(stage_chunk)
        p.group_cols = int(group_cols)
        p.check_owners = int(check_owners)
        p.grid_cols = int(grid_cols)
        p.q_cache = int(q_cache)
        p.lr_rule, p.ada_eps = {"eq9": 0, "adagrad": 1}[lr_rule], ada_eps
        p.device, p.rank, p.world, p.transport = device, rank, world, transport
        self._id_buf = None
        if nccl_id is not None:
            self._id_buf = ctypes.create_string_buffer(bytes(nccl_id), 128)
            p.nccl_id = ctypes.cast(self._id_buf, ctypes.c_void_p)
        torch = _torch()
        if stream is None and torch.cuda.is_available():
            stream = torch.cuda.current_stream(device)
        if stream is not None:
            p.stream = ctypes.c_void_p(int(getattr(stream, "cuda_stream", stream)) or None)
        self._alloc = None
        if allocator == "torch" and torch.cuda.is_available():
            self._alloc = _TorchAllocator(device, device_budget)
            p.alloc = ctypes.pointer(self._alloc.struct)
        self.params = p
        self.m, self.n, self.k = int(m), int(n), int(k)
        self.device = device
        h = ctypes.c_void_p()
        st = L.mf_create(ctypes.byref(p), ctypes.byref(h))
        if st != 0:
            raise MFError(st, "mf_create")
        self.h = h

    # -- helpers
    def _check(self, st: int, what: str):
        if st != 0:
            msg = lib().mf_last_error(self.h)
            raise MFError(st, f"{what}: {msg.decode() if msg else ''}")

    def close(self):
        if getattr(self, "h", None):
            lib().mf_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # -- API
    def load(self, u, v, r, set: str = "train", on_device: bool | None = None):
        if on_device is None:
            on_device = _is_cuda_tensor(u)
        pu, ku = _as_ptr(u, np.int32, on_device)
        pv, kv = _as_ptr(v, np.int32, on_device)
        pr, kr = _as_ptr(r, np.float32, on_device)
        n = len(ku)
        self._check(lib().mf_load_coo(self.h, SETS[set], n, pu, pv, pr, int(on_device)),
                    f"mf_load_coo({set})")

    def train_epoch(self) -> int:
        t = ctypes.c_int32(0)
        self._check(lib().mf_train_epoch(self.h, ctypes.byref(t)), "mf_train_epoch")
        return t.value

    def rmse(self, set: str = "test") -> float:
        out = ctypes.c_double(0)
        self._check(lib().mf_rmse(self.h, SETS[set], ctypes.byref(out)), "mf_rmse")
        return out.value

    def loss(self) -> float:
        """Eq. 2 over the training set (scaled rating units)."""
        out = ctypes.c_double(0)
        self._check(lib().mf_loss(self.h, ctypes.byref(out)), "mf_loss")
        return out.value

    def factors(self, on_device: bool = False):
        if on_device:
            torch = _torch()
            P = torch.empty((self.m, self.k), dtype=torch.float32, device=f"cuda:{self.device}")
            Q = torch.empty((self.n, self.k), dtype=torch.float32, device=f"cuda:{self.device}")
            self._check(lib().mf_get_factors(self.h, ctypes.c_void_p(P.data_ptr()),
                                             ctypes.c_void_p(Q.data_ptr()), 1), "mf_get_factors")
            return P, Q
        P = np.empty((self.m, self.k), dtype=np.float32)
        Q = np.empty((self.n, self.k), dtype=np.float32)
        self._check(lib().mf_get_factors(self.h, P.ctypes.data, Q.ctypes.data, 0), "mf_get_factors")
        return P, Q

    def set_factors(self, P=None, Q=None):
        P = None if P is None else np.ascontiguousarray(P, dtype=np.float32)
        Q = None if Q is None else np.ascontiguousarray(Q, dtype=np.float32)
        self._check(lib().mf_set_factors(self.h, None if P is None else P.ctypes.data,
                                         None if Q is None else Q.ctypes.data, 0), "mf_set_factors")

    @property
    def epoch(self) -> int:
        t = ctypes.c_int32(0)
        self._check(lib().mf_get_epoch(self.h, ctypes.byref(t)), "mf_get_epoch")
        return t.value

    def set_epoch(self, t: int):
        self._check(lib().mf_set_epoch(self.h, t), "mf_set_epoch")

    def export(self, what: str, epoch: int = 0) -> np.ndarray:
        n = ctypes.c_int64(0)
        self._check(lib().mf_export_schedule(self.h, EXPORTS[what], epoch, None, ctypes.byref(n)),
                    f"export({what})")
        buf = np.empty(max(n.value, 1), dtype=np.int64)
        self._check(lib().mf_export_schedule(self.h, EXPORTS[what], epoch, buf.ctypes.data,
                                             ctypes.byref(n)), f"export({what})")
        return buf[:n.value]

    def launch_ms(self) -> np.ndarray:
        """Device time (ms) of each SGD launch of the last epoch, in launch order."""
        n = ctypes.c_int64(0)
        self._check(lib().mf_get_launch_ms(self.h, None, ctypes.byref(n)), "mf_get_launch_ms")
        buf = np.zeros(max(n.value, 1), dtype=np.float64)
        self._check(lib().mf_get_launch_ms(self.h, buf.ctypes.data, ctypes.byref(n)),
                    "mf_get_launch_ms")
        return buf[:n.value]

    def check_visits(self) -> dict:
        """Exactly-once evidence from the device (mf_check_visits): work units whose claim count
        differs from the epochs run since load."""
        bad, units, ep = ctypes.c_int64(0), ctypes.c_int64(0), ctypes.c_int32(0)
        self._check(lib().mf_check_visits(self.h, ctypes.byref(bad), ctypes.byref(units),
                                          ctypes.byref(ep)), "mf_check_visits")
        return {"bad_units": bad.value, "units": units.value, "epochs": ep.value}

    @property
    def device_peak_bytes(self) -> int:
        """High-water mark of the ctx's device memory (torch allocator hooks only)."""
        return self._alloc.peak if self._alloc is not None else -1

    def owner_violations(self) -> int:
        """Ownership-checker violations since load (check_owners = True, wavefront)."""
        n = ctypes.c_int64(0)
        self._check(lib().mf_owner_violations(self.h, ctypes.byref(n)), "mf_owner_violations")
        return n.value

    def stats(self) -> dict:
        s = Stats()
        self._check(lib().mf_get_stats(self.h, ctypes.byref(s)), "mf_get_stats")
        return {name: getattr(s, name) for name, _ in Stats._fields_}


# ---------------------------------------------------------------------------------------------
# The C ABI's own names (include/mf.h), function style: each forwards to the MF method or the
# library call above (argument marshalling only).
# ---------------------------------------------------------------------------------------------
def mf_abi_version() -> int:
    return int(lib().mf_abi_version())


def mf_status_string(status: int) -> str:
    return lib().mf_status_string(int(status)).decode()


def mf_params_default() -> Params:
    p = Params()
    lib().mf_params_default(ctypes.byref(p))
    return p


def mf_create(m: int, n: int, k: int = 128, **params) -> MF:
    return MF(m, n, k, **params)


def mf_load_coo(ctx: MF, set: str, u, v, r, on_device: bool | None = None) -> None:
    ctx.load(u, v, r, set, on_device)


def mf_train_epoch(ctx: MF) -> int:
    return ctx.train_epoch()


def mf_rmse(ctx: MF, set: str = "test") -> float:
    return ctx.rmse(set)


def mf_loss(ctx: MF) -> float:
    return ctx.loss()


def mf_get_factors(ctx: MF, on_device: bool = False):
    return ctx.factors(on_device)


def mf_set_factors(ctx: MF, P=None, Q=None) -> None:
    ctx.set_factors(P, Q)


def mf_get_epoch(ctx: MF) -> int:
    return ctx.epoch


def mf_set_epoch(ctx: MF, t: int) -> None:
    ctx.set_epoch(t)


def mf_export_schedule(ctx: MF, what: str, epoch: int = 0) -> np.ndarray:
    return ctx.export(what, epoch)


def mf_get_stats(ctx: MF) -> dict:
    return ctx.stats()


def mf_get_launch_ms(ctx: MF) -> np.ndarray:
    return ctx.launch_ms()


def mf_check_visits(ctx: MF) -> dict:
    return ctx.check_visits()


def mf_owner_violations(ctx: MF) -> int:
    return ctx.owner_violations()


def mf_last_error(ctx: MF) -> str:
    msg = lib().mf_last_error(ctx.h)
    return msg.decode() if msg else ""


def mf_destroy(ctx: MF) -> None:
    ctx.close()


mf_strata_holders = strata_holders
mf_strata_plan = strata_plan
mf_comm_selftest = comm_selftest


def _is_cuda_tensor(x) -> bool:
    try:
        import torch
        return isinstance(x, torch.Tensor) and x.is_cuda
    except ImportError:
        return False


def nccl_unique_id_via(group=None) -> bytes:
    """Create an ncclUniqueId on rank 0 and broadcast it over torch.distributed (gloo or nccl)."""
    torch = _torch()
    import torch.distributed as dist
    if dist.get_rank(group) == 0:
        uid = _nccl_get_unique_id()
        t = torch.tensor(list(uid), dtype=torch.uint8)
    else:
        t = torch.zeros(128, dtype=torch.uint8)
    if dist.get_backend(group) == "nccl":
        t = t.cuda()
    dist.broadcast(t, src=0, group=group)
    return bytes(t.cpu().tolist())


def _nccl_get_unique_id() -> bytes:
    for name in ("libnccl.so.2", "libnccl.so"):
        try:
            L = ctypes.CDLL(name, mode=ctypes.RTLD_GLOBAL)
            break
        except OSError:
            L = None
    if L is None:
        raise MFError(-4, "libnccl.so.2 not loadable")
    buf = ctypes.create_string_buffer(128)
    st = L.ncclGetUniqueId(buf)
    if st != 0:
        raise MFError(-4, f"ncclGetUniqueId -> {st}")
    return buf.raw
