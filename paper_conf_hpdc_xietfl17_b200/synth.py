"""Seeded synthetic rating generators (the ONE module both the oracle and the CUDA path consume).

Holds none of the method's arithmetic: it only draws COO ratings (u, v, r) with the shapes
of Table 2 and the recipe stated in DESIGN.md section 4:

* rows u ~ inverse-CDF of weights (rank+1)^-a_u over a seeded random relabelling of row ids,
  columns v likewise with a_v (Chung-Lu bipartite, u and v independent);
* r = mu + p*_u . q*_v + eps, planted rank r* (entries N(0,1)/r*^(1/4), signal variance ~1),
  eps ~ N(0, noise^2); the Yahoo-shaped set uses r = 50 + 25 (p*.q* + eps) clipped to [0, 100];
* the test set is drawn iid from the same process with its own stream (seed + 100) (R17).

Large sets are generated with torch on whatever device is given (CUDA on the GPU box), in
chunks, so that 99M - 3.1B samples stay tractable.  The generator is counter-based: the same
seed gives bit-identical data on the CPU and on the GPU (so oracle reference values can be
computed on a CPU box and compared with a GPU run).  The tiny set uses numpy.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import torch

# Table 2 and Table 3
SHAPES = {
    "netflix": dict(m=480_190, n=17_771, N=99_072_112, Ntest=1_408_395,
                    lam=0.05, alpha=0.08, beta=0.3, mu=3.6, scale="plain", rating_scale=1.0,
                    data_seed=1),
    "yahoo": dict(m=1_000_990, n=624_961, N=252_800_275, Ntest=4_003_960,
                  lam=1.0, alpha=0.08, beta=0.2, mu=50.0, scale="yahoo", rating_scale=25.0,
                  data_seed=2),
    # Hugewiki-shaped ratings are CENTERED (mu = 0; R22): with mu = 3.6 the serial
    # oracle itself diverges under Table 3's alpha at this m/n (NaN after one epoch at 5% scale).
    "hugewiki": dict(m=50_082_604, n=39_781, N=3_069_817_980, Ntest=31_327_899,
                     lam=0.03, alpha=0.08, beta=0.3, mu=0.0, scale="plain", rating_scale=1.0,
                     data_seed=3),
}


@dataclass
class Ratings:
    m: int
    n: int
    u: object          # int32 array / tensor
    v: object
    r: object          # float32
    ut: object = None  # test set
    vt: object = None
    rt: object = None
    meta: dict = field(default_factory=dict)

    @property
    def N(self) -> int:
        return int(len(self.u))

    @property
    def Ntest(self) -> int:
        return 0 if self.ut is None else int(len(self.ut))


def tiny(seed: int = 0, m: int = 1000, n: int = 800, N: int = 50_000, Ntest: int = 5_000,
         rank: int = 4) -> Ratings:
    """configs[0]: planted rank-4, noiseless, uniform UNIQUE (u,v) pairs."""
    rng = np.random.default_rng(seed)
    cells = rng.choice(m * n, size=N + Ntest, replace=False)
    u = (cells // n).astype(np.int32)
    v = (cells % n).astype(np.int32)
    Ps = rng.standard_normal((m, rank)) / rank ** 0.25
    Qs = rng.standard_normal((n, rank)) / rank ** 0.25
    r = np.einsum("ij,ij->i", Ps[u], Qs[v]).astype(np.float32)
    return Ratings(m, n, u[:N], v[:N], r[:N], u[N:], v[N:], r[N:],
                   meta=dict(kind="tiny-planted", rank=rank, seed=seed, unique=True))


def uniform(m: int, n: int, N: int, seed: int = 0, mu: float = 0.0, rank: int = 4,
            noise: float = 0.0, Ntest: int = 0) -> Ratings:
    """Uniform (u, v) with duplicates allowed (R18), planted low rank plus noise."""
    rng = np.random.default_rng(seed)
    Ps = rng.standard_normal((m, rank)) / rank ** 0.25
    Qs = rng.standard_normal((n, rank)) / rank ** 0.25

    def draw(cnt):
        u = rng.integers(0, m, cnt).astype(np.int32)
        v = rng.integers(0, n, cnt).astype(np.int32)
        r = (mu + np.einsum("ij,ij->i", Ps[u], Qs[v]) + noise * rng.standard_normal(cnt))
        return u, v, r.astype(np.float32)

    u, v, r = draw(N)
    ut, vt, rt = draw(Ntest) if Ntest else (None, None, None)
    return Ratings(m, n, u, v, r, ut, vt, rt, meta=dict(kind="uniform", seed=seed))


# ---------------------------------------------------------------------------------------------
# Counter-based draws (device independent).  Every random number is a pure function of
# (data seed, stream tag, global index): a 64-bit hash of the index, evaluated with int64
# tensor arithmetic (two's-complement wrap-around, logical shifts by masking) on whatever device
# the tensors live on.  Every float derived from it is built from exact integer-to-float
# conversions and single IEEE operations (no transcendental functions, no fused or reordered
# reductions), so CPU and CUDA produce the SAME bits for the same seed -- tests/test_synth.py
# pins the hash against a plain-Python rendering and CPU against CUDA.  The hash is MurmurHash3's
# 64-bit finaliser (fmix64) of seed-keyed counters; it is deliberately not the method's own
# SplitMix64 key function, which this module does not contain.
# ---------------------------------------------------------------------------------------------
_M64 = 1 << 64
_F1, _F2 = 0xFF51AFD7ED558CCD, 0xC4CEB9FE1A85EC53          # fmix64 constants
_GOLD = 0x9E3779B97F4A7C15                                   # Weyl increment of the counter


def _s64(c: int) -> int:
    """A uint64 constant as the int64 with the same bits."""
    c %= _M64
    return c - _M64 if c >= 1 << 63 else c


def _shr(z: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (z >> s) & ((1 << (64 - s)) - 1)


def fmix64(z: torch.Tensor) -> torch.Tensor:
    z = z ^ _shr(z, 33)
    z = z * _s64(_F1)
    z = z ^ _shr(z, 33)
    z = z * _s64(_F2)
    return z ^ _shr(z, 33)


def fmix64_int(z: int) -> int:
    """Plain-Python fmix64 (the pin of the tensor version; also derives stream keys)."""
    z %= _M64
    z ^= z >> 33
    z = (z * _F1) % _M64
    z ^= z >> 33
    z = (z * _F2) % _M64
    return z ^ (z >> 33)


def stream_key(seed: int, tag: int) -> int:
    return fmix64_int(fmix64_int(seed * _GOLD + 1) + tag * _GOLD)


def hash_at(key: int, idx: torch.Tensor) -> torch.Tensor:
    """64-bit hash (int64 bits) of counters idx (int64) under a stream key."""
    return fmix64(idx * _s64(_GOLD) + _s64(key))


def uniform53(key: int, idx: torch.Tensor) -> torch.Tensor:
    """U[0,1) in float64 with 53 random bits (exact conversion)."""
    return _shr(hash_at(key, idx), 11).to(torch.float64) * (2.0 ** -53)


def normal_ih(key: int, idx: torch.Tensor) -> torch.Tensor:
    """Approximately N(0,1): Irwin-Hall sum of 12 U24 uniforms minus 6 (six hashes, two 24-bit
    uniforms each).  Every partial sum is exact in float64 (< 2^28 units of 2^-24), so the
    result does not depend on the order of evaluation or the device."""
    acc = torch.zeros(idx.shape, dtype=torch.float64, device=idx.device)
    for j in range(6):
        h = hash_at(key, idx * 6 + j)
        acc += _shr(h, 40).to(torch.float64) * (2.0 ** -24)
        acc += (_shr(h, 16) & 0xFFFFFF).to(torch.float64) * (2.0 ** -24)
    return acc - 6.0


def _cdf(size: int, expo: float) -> np.ndarray:
    """Normalised CDF of weights (rank+1)^-expo, computed once on the host in float64 (the
    only place a pow() is evaluated) and shipped to the device bit for bit."""
    w = np.arange(1, size + 1, dtype=np.float64) ** (-expo)
    c = np.cumsum(w)
    return c / c[-1]


# stream tags of the recipe
_T_RELAB_U, _T_RELAB_V, _T_PS, _T_QS, _T_U, _T_V, _T_EPS = 1, 2, 3, 4, 5, 6, 7
_TEST_SEED_OFFSET = 100       # R17: the test set is the same process on seed + 100


def powerlaw(m: int, n: int, N: int, Ntest: int, *, seed: int, a_u: float = 0.38,
             a_v: float = 0.45, rank: int = 16, mu: float = 3.6, noise: float = 0.5,
             scale: str = "plain", device="cpu", chunk: int = 1 << 24,
             out_device=None) -> Ratings:
    """Power-law-skewed planted-rank ratings (SURVEY 8(d) recipe),
    counter-based: the same (m, n, N, seed, ...) gives bit-identical (u, v, r) on any device and
    for any chunk size."""
    dev = torch.device(device)
    out_dev = dev if out_device is None else torch.device(out_device)
    cdf_u = torch.from_numpy(_cdf(m, a_u)).to(dev)
    cdf_v = torch.from_numpy(_cdf(n, a_v)).to(dev)

    def relabel(size, tag):   # a uniformly random permutation of the ids: argsort of distinct keys
        k = hash_at(stream_key(seed, tag), torch.arange(size, dtype=torch.int64, device=dev))
        return torch.argsort(k).to(torch.int32)

    relab_u, relab_v = relabel(m, _T_RELAB_U), relabel(n, _T_RELAB_V)
    amp = 1.0 / rank ** 0.25

    def factors(size, tag):   # planted factors, entries ~ N(0,1) / rank^(1/4), float32
        out = torch.empty(size, rank, dtype=torch.float32, device=dev)
        for lo in range(0, size, chunk // rank):
            c = min(chunk // rank, size - lo)
            idx = torch.arange(lo * rank, (lo + c) * rank, dtype=torch.int64, device=dev)
            out[lo:lo + c] = (normal_ih(stream_key(seed, tag), idx) * amp).to(torch.float32).view(c, rank)
        return out

    Ps, Qs = factors(m, _T_PS), factors(n, _T_QS)

    def ids(key, idx, size, cdf, relab):
        x = uniform53(key, idx)
        return relab[torch.searchsorted(cdf, x).clamp_(max=size - 1)]

    def draw(cnt, sd):
        ku, kv, ke = stream_key(sd, _T_U), stream_key(sd, _T_V), stream_key(sd, _T_EPS)
        u = torch.empty(cnt, dtype=torch.int32, device=out_dev)
        v = torch.empty(cnt, dtype=torch.int32, device=out_dev)
        r = torch.empty(cnt, dtype=torch.float32, device=out_dev)
        for lo in range(0, cnt, chunk):
            c = min(chunk, cnt - lo)
            idx = torch.arange(lo, lo + c, dtype=torch.int64, device=dev)
            uu = ids(ku, idx, m, cdf_u, relab_u)
            vv = ids(kv, idx, n, cdf_v, relab_v)
            pu, qv = Ps[uu.long()], Qs[vv.long()]
            sig = torch.zeros(c, dtype=torch.float64, device=dev)
            for d in range(rank):     # separate IEEE multiply and add: no contraction, fixed order
                sig = sig + pu[:, d].to(torch.float64) * qv[:, d].to(torch.float64)
            eps = normal_ih(ke, idx) * noise
            if scale == "yahoo":
                rr = (50.0 + 25.0 * (sig + eps)).clamp_(0.0, 100.0)
            else:
                rr = mu + sig + eps
            u[lo:lo + c] = uu.to(out_dev)
            v[lo:lo + c] = vv.to(out_dev)
            r[lo:lo + c] = rr.to(torch.float32).to(out_dev)
        return u, v, r

    u, v, r = draw(N, seed)
    ut, vt, rt = draw(Ntest, seed + _TEST_SEED_OFFSET) if Ntest else (None, None, None)
    meta = dict(kind="powerlaw-counter", seed=seed, a_u=a_u, a_v=a_v, rank=rank, mu=mu,
                noise=noise, scale=scale)
    return Ratings(m, n, u, v, r, ut, vt, rt, meta=meta)


def checksum(R: Ratings) -> str:
    """Order-sensitive 64-bit digest of (u, v, r-bits) of the train and test sets (hex), for
    pinning a generated set across devices (golden files carry it)."""
    tot = 0
    for arr in (R.u, R.v, R.r, R.ut, R.vt, R.rt):
        if arr is None:
            continue
        t = torch.as_tensor(arr)
        t = (t.view(torch.int32) if t.dtype == torch.float32 else t.to(torch.int32)).to(torch.int64)
        idx = torch.arange(t.numel(), dtype=torch.int64, device=t.device)
        h = hash_at(0x5EED, idx * 2 + (t & 0xFFFFFFFF))
        part = int((h & 0xFFFFFFFF).sum().item()) + (int((_shr(h, 32)).sum().item()) << 32)
        tot = fmix64_int(tot + part)
    return f"{tot:016x}"


def shaped(name: str, *, fraction: float = 1.0, device="cpu", out_device=None,
           with_test: bool = True) -> Ratings:
    """A Table-2-shaped set; `fraction` < 1 scales m, n, N, Ntest together (tests)."""
    s = SHAPES[name]
    m = max(16, int(s["m"] * fraction))
    n = max(16, int(s["n"] * fraction))
    N = max(1, int(s["N"] * fraction))
    Nt = max(1, int(s["Ntest"] * fraction)) if with_test else 0
    R = powerlaw(m, n, N, Nt, seed=s["data_seed"], mu=s["mu"], scale=s["scale"],
                 device=device, out_device=out_device)
    R.meta.update(name=name, fraction=fraction)
    return R


def degree_stats(R: Ratings) -> dict:
    """max / mean row and column degree of the training set (the manifest SURVEY 8(d) asks for)."""
    u = torch.as_tensor(R.u)
    v = torch.as_tensor(R.v)
    du = torch.bincount(u.long(), minlength=R.m)
    dv = torch.bincount(v.long(), minlength=R.n)
    return dict(max_row_deg=int(du.max()), mean_row_deg=float(R.N / R.m),
                max_col_deg=int(dv.max()), mean_col_deg=float(R.N / R.n))
