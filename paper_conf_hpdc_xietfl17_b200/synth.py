"""Seeded synthetic rating generators (the ONE module both the oracle and the CUDA path consume).

Holds none of the method's arithmetic: it only draws COO ratings (u, v, r) with the shapes
of Table 2 and the recipe stated in DESIGN.md section 4:

* rows u ~ inverse-CDF of weights (rank+1)^-a_u over a seeded random relabelling of row ids,
  columns v likewise with a_v (Chung-Lu bipartite, u and v independent);
* r = mu + p*_u . q*_v + eps, planted rank r* (entries N(0,1)/r*^(1/4), signal variance ~1),
  eps ~ N(0, noise^2); the Yahoo-shaped set uses r = 50 + 25 (p*.q* + eps) clipped to [0, 100];
* the test set is drawn iid from the same process with its own stream (seed + 100) (R17).

Large sets are generated with torch on whatever device is given (CUDA on the GPU box), in
chunks, so that 99M - 3.1B samples stay tractable; the tiny set uses numpy.
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


def _powerlaw_ids(count: int, size: int, expo: float, relabel: torch.Tensor,
                  cdf: torch.Tensor, g: torch.Generator, device) -> torch.Tensor:
    x = torch.rand(count, generator=g, device=device, dtype=torch.float64)
    rank = torch.searchsorted(cdf, x).clamp_(max=size - 1)
    return relabel[rank].to(torch.int32)


def powerlaw(m: int, n: int, N: int, Ntest: int, *, seed: int, a_u: float = 0.38,
             a_v: float = 0.45, rank: int = 16, mu: float = 3.6, noise: float = 0.5,
             scale: str = "plain", device="cpu", chunk: int = 1 << 24,
             out_device=None) -> Ratings:
    """Power-law-skewed planted-rank ratings (SURVEY 8(d) recipe), generated in chunks."""
    dev = torch.device(device)
    out_dev = dev if out_device is None else torch.device(out_device)
    g = torch.Generator(device=dev)
    g.manual_seed(seed)

    def cdf_of(size, expo):
        w = torch.arange(1, size + 1, device=dev, dtype=torch.float64).pow_(-expo)
        c = torch.cumsum(w, 0)
        return c / c[-1]

    cdf_u, cdf_v = cdf_of(m, a_u), cdf_of(n, a_v)
    relab_u = torch.randperm(m, generator=g, device=dev)
    relab_v = torch.randperm(n, generator=g, device=dev)
    Ps = torch.randn(m, rank, generator=g, device=dev) / rank ** 0.25
    Qs = torch.randn(n, rank, generator=g, device=dev) / rank ** 0.25

    def draw(cnt, gen):
        u = torch.empty(cnt, dtype=torch.int32, device=out_dev)
        v = torch.empty(cnt, dtype=torch.int32, device=out_dev)
        r = torch.empty(cnt, dtype=torch.float32, device=out_dev)
        for lo in range(0, cnt, chunk):
            c = min(chunk, cnt - lo)
            uu = _powerlaw_ids(c, m, a_u, relab_u, cdf_u, gen, dev)
            vv = _powerlaw_ids(c, n, a_v, relab_v, cdf_v, gen, dev)
            sig = (Ps[uu.long()] * Qs[vv.long()]).sum(1)
            eps = torch.randn(c, generator=gen, device=dev) * noise
            if scale == "yahoo":
                rr = (50.0 + 25.0 * (sig + eps)).clamp_(0.0, 100.0)
            else:
                rr = mu + sig + eps
            u[lo:lo + c] = uu.to(out_dev)
            v[lo:lo + c] = vv.to(out_dev)
            r[lo:lo + c] = rr.to(torch.float32).to(out_dev)
        return u, v, r

    u, v, r = draw(N, g)
    gt = torch.Generator(device=dev)
    gt.manual_seed(seed + 100)
    ut, vt, rt = draw(Ntest, gt) if Ntest else (None, None, None)
    meta = dict(kind="powerlaw", seed=seed, a_u=a_u, a_v=a_v, rank=rank, mu=mu, noise=noise,
                scale=scale)
    return Ratings(m, n, u, v, r, ut, vt, rt, meta=meta)


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
