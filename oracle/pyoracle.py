"""ctypes wrapper of oracle/liboracle.so (plain C, single-threaded CPU oracle).

TEST INFRASTRUCTURE ONLY: only tests/, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this module.  The product package
``paper_conf_hpdc_xietfl17_b200`` never imports it.  See oracle/oracle.h for the contract
and the paper passages each function follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "oracle.c")
HDR = os.path.join(HERE, "oracle.h")
LIB = os.path.join(HERE, "liboracle.so")

STORAGE = {"fp32": 0, "fp16": 1, "bf16": 2}
SCHEDULE = {"hogwild": 0, "wavefront": 1}
EX = {"perm": 0, "rho_r": 1, "rho_c": 2, "blockid": 3, "chunkorder": 4, "wfseq": 5,
      "tickets": 6, "strata": 7, "order": 8}


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-O2, no FMA contraction)."""
    stale = (not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(SRC),
                                                                     os.path.getmtime(HDR)))
    if force or stale:
        subprocess.run(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fPIC", "-shared",
                        "-Wall", SRC, "-o", LIB, "-lm"], check=True)
    return LIB


class Params(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("n", ctypes.c_int64), ("k", ctypes.c_int32),
                ("lambda_p", ctypes.c_float), ("lambda_q", ctypes.c_float),
                ("alpha", ctypes.c_float), ("beta", ctypes.c_float),
                ("init_scale", ctypes.c_float), ("rating_scale", ctypes.c_float),
                ("seed", ctypes.c_uint64), ("schedule", ctypes.c_int32),
                ("storage", ctypes.c_int32), ("workers", ctypes.c_int32),
                ("batch_f", ctypes.c_int32), ("wf_cols", ctypes.c_int32),
                ("grid_a", ctypes.c_int32), ("cyclic", ctypes.c_int32),
                ("lr_rule", ctypes.c_int32), ("ada_eps", ctypes.c_float),
                ("group_cols", ctypes.c_int32), ("grid_cols", ctypes.c_int32)]


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        u64, i64, i32, f32, f64 = (ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32,
                                   ctypes.c_float, ctypes.c_double)
        vp = ctypes.c_void_p
        sig = {
            "or_mix": (u64, [u64]), "or_stream": (u64, [u64, u64, u64, u64]),
            "or_key": (u64, [u64, u64]), "or_perm": (ctypes.c_int, [u64, i64, vp]),
            "or_f16_bits": (ctypes.c_uint16, [f32]), "or_f16_value": (f32, [ctypes.c_uint16]),
            "or_bf16_bits": (ctypes.c_uint16, [f32]), "or_bf16_value": (f32, [ctypes.c_uint16]),
            "or_round_storage": (f32, [i32, f32]), "or_gamma": (f32, [f32, f32, i32]),
            "or_update": (None, [i32, vp, vp, f32, f32, f32, f32, i32]),
            "or_update_adagrad": (None, [i32, vp, vp, vp, vp, f32, f32, f32, f32, f32, i32]),
            "or_sample_loss": (f64, [i32, vp, vp, f64, f64, f64]),
            "or_create": (vp, [ctypes.POINTER(Params), i64, vp, vp, vp]),
            "or_destroy": (None, [vp]), "or_train_epoch": (ctypes.c_int, [vp]),
            "or_run_block": (ctypes.c_int, [vp, i32, i64]),
            "or_set_epoch": (ctypes.c_int, [vp, i32]), "or_get_epoch": (i32, [vp]),
            "or_rmse": (f64, [vp, i64, vp, vp, vp]), "or_loss": (f64, [vp]),
            "or_get_factors": (None, [vp, vp, vp]), "or_set_factors": (None, [vp, vp, vp]),
            "or_copy_q_rows": (None, [vp, vp, i64, i64]),
            "or_export": (ctypes.c_int, [vp, i32, i32, vp, ctypes.POINTER(i64)]),
        }
        for name, (res, args) in sig.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def perm(S: int, n: int) -> np.ndarray:
    out = np.empty(max(n, 1), dtype=np.int64)
    assert lib().or_perm(S, n, _ptr(out)) == 0
    return out[:n]


def update(p, q, r, gamma, lambda_p, lambda_q, storage="fp32"):
    """One Algorithm-1 update on copies of p, q (float32); returns (p', q')."""
    p = np.array(p, dtype=np.float32).copy()
    q = np.array(q, dtype=np.float32).copy()
    lib().or_update(len(p), _ptr(p), _ptr(q), r, gamma, lambda_p, lambda_q, STORAGE[storage])
    return p, q


def update_adagrad(p, q, gp, gq, r, alpha, lambda_p, lambda_q, eps=1e-8, storage="fp32"):
    """One ADAGRAD update (R23) on copies; returns (p', q', gp', gq')."""
    p, q, gp, gq = (np.array(x, dtype=np.float32).copy() for x in (p, q, gp, gq))
    lib().or_update_adagrad(len(p), _ptr(p), _ptr(q), _ptr(gp), _ptr(gq), r, alpha, lambda_p,
                            lambda_q, eps, STORAGE[storage])
    return p, q, gp, gq


def sample_loss(p, q, r, lambda_p, lambda_q) -> float:
    p = np.ascontiguousarray(p, dtype=np.float64)
    q = np.ascontiguousarray(q, dtype=np.float64)
    return lib().or_sample_loss(len(p), _ptr(p), _ptr(q), r, lambda_p, lambda_q)


class Oracle:
    """One oracle training run (Alg. 1 with the chosen serial schedule)."""

    def __init__(self, m, n, k, u, v, r, *, lambda_p=0.05, lambda_q=None, alpha=0.08, beta=0.3,
                 init_scale=1.0, rating_scale=1.0, seed=42, schedule="hogwild", storage="fp32",
                 workers=1, batch_f=256, wf_cols=0, grid_a=1, cyclic=False, lr_rule="eq9",
                 ada_eps=1e-8, group_cols=False, grid_cols=0):
        self.m, self.n, self.k = int(m), int(n), int(k)
        self.p = Params(m=m, n=n, k=k, lambda_p=lambda_p,
                        lambda_q=lambda_p if lambda_q is None else lambda_q, alpha=alpha,
                        beta=beta, init_scale=init_scale, rating_scale=rating_scale, seed=seed,
                        schedule=SCHEDULE[schedule], storage=STORAGE[storage], workers=workers,
                        batch_f=batch_f, wf_cols=wf_cols, grid_a=grid_a, cyclic=int(cyclic),
                        lr_rule={"eq9": 0, "adagrad": 1}[lr_rule], ada_eps=ada_eps,
                        group_cols=int(group_cols), grid_cols=int(grid_cols))
        self.u = np.ascontiguousarray(u, dtype=np.int32)
        self.v = np.ascontiguousarray(v, dtype=np.int32)
        self.r = np.ascontiguousarray(r, dtype=np.float32)
        self.N = len(self.u)
        self.h = lib().or_create(ctypes.byref(self.p), self.N, _ptr(self.u), _ptr(self.v),
                                 _ptr(self.r))
        if not self.h:
            raise ValueError("or_create rejected its input")

    def __del__(self):
        h = getattr(self, "h", None)
        if h:
            lib().or_destroy(h)
            self.h = None

    def train_epoch(self) -> None:
        assert lib().or_train_epoch(self.h) == 0

    def run_block(self, t: int, b: int) -> None:
        assert lib().or_run_block(self.h, t, b) == 0

    def set_epoch(self, t: int) -> None:
        assert lib().or_set_epoch(self.h, t) == 0

    @property
    def epoch(self) -> int:
        return lib().or_get_epoch(self.h)

    def rmse(self, u, v, r) -> float:
        u = np.ascontiguousarray(u, dtype=np.int32)
        v = np.ascontiguousarray(v, dtype=np.int32)
        r = np.ascontiguousarray(r, dtype=np.float32)
        return lib().or_rmse(self.h, len(u), _ptr(u), _ptr(v), _ptr(r))

    def loss(self) -> float:
        return lib().or_loss(self.h)

    def factors(self):
        P = np.empty((self.m, self.k), dtype=np.float32)
        Q = np.empty((self.n, self.k), dtype=np.float32)
        lib().or_get_factors(self.h, _ptr(P), _ptr(Q))
        return P, Q

    def set_factors(self, P=None, Q=None) -> None:
        P = None if P is None else np.ascontiguousarray(P, dtype=np.float32)
        Q = None if Q is None else np.ascontiguousarray(Q, dtype=np.float32)
        lib().or_set_factors(self.h, None if P is None else _ptr(P),
                             None if Q is None else _ptr(Q))

    def copy_q_rows_from(self, other: "Oracle", lo: int, hi: int) -> None:
        lib().or_copy_q_rows(self.h, other.h, lo, hi)

    def export(self, what: str, t: int = 0) -> np.ndarray:
        n = ctypes.c_int64(0)
        assert lib().or_export(self.h, EX[what], t, None, ctypes.byref(n)) == 0
        buf = np.empty(max(n.value, 1), dtype=np.int64)
        assert lib().or_export(self.h, EX[what], t, _ptr(buf), ctypes.byref(n)) == 0
        return buf[:n.value]
