"""The shared input generator (synth.py) is counter-based and device independent.

It holds none of the method's arithmetic; these tests pin its hash against a plain-Python
rendering, its draws against their distributions (DESIGN.md section 4 recipe), and (-m gpu)
the CUDA rendering against the CPU one bit for bit -- which is what lets tests/golden/ hold
oracle values computed on a CPU box for data the GPU tests generate on the device.
"""
import numpy as np
import pytest
import torch

from paper_conf_hpdc_xietfl17_b200 import synth


def test_fmix64_tensor_equals_plain_python():
    rng = np.random.default_rng(0)
    vals = [0, 1, 2, (1 << 63) - 1, -(1 << 63), -1, 0x1234567890ABCDEF]
    vals += [int(x) for x in rng.integers(-(1 << 63), (1 << 63) - 1, 2000, dtype=np.int64)]
    t = synth.fmix64(torch.tensor(vals, dtype=torch.int64))
    for x, h in zip(vals, t.tolist()):
        assert h % (1 << 64) == synth.fmix64_int(x % (1 << 64))
    # fmix64 is a bijection with fmix64(0) = 0 (MurmurHash3)
    assert synth.fmix64_int(0) == 0


def test_hash_at_matches_definition():
    key = synth.stream_key(7, 3)
    idx = torch.arange(0, 5000, 7, dtype=torch.int64)
    h = synth.hash_at(key, idx)
    for i, x in zip(idx.tolist(), h.tolist()):
        assert x % (1 << 64) == synth.fmix64_int(i * synth._GOLD + key)


def test_uniform_and_irwin_hall_moments():
    idx = torch.arange(1 << 20, dtype=torch.int64)
    u = synth.uniform53(synth.stream_key(1, 1), idx)
    assert float(u.min()) >= 0.0 and float(u.max()) < 1.0
    assert abs(float(u.mean()) - 0.5) < 2e-3 and abs(float(u.var()) - 1 / 12) < 1e-3
    z = synth.normal_ih(synth.stream_key(1, 2), idx)
    assert abs(float(z.mean())) < 5e-3 and abs(float(z.var()) - 1.0) < 5e-3
    assert float(z.abs().max()) <= 6.0


def test_powerlaw_is_chunk_independent_and_shaped():
    kw = dict(seed=5, rank=8, mu=3.6, noise=0.5)
    a = synth.powerlaw(4000, 900, 200_000, 20_000, **kw)
    b = synth.powerlaw(4000, 900, 200_000, 20_000, chunk=1 << 13, **kw)
    assert synth.checksum(a) == synth.checksum(b)
    for x, y in ((a.u, b.u), (a.v, b.v), (a.r, b.r), (a.ut, b.ut), (a.rt, b.rt)):
        assert torch.equal(x, y)
    assert int(a.u.min()) >= 0 and int(a.u.max()) < 4000 and int(a.v.max()) < 900
    # the heaviest column's share follows the recipe's weights (rank+1)^-0.45 (relabelled)
    w = np.arange(1, 901, dtype=np.float64) ** -0.45
    share = np.bincount(a.v.numpy(), minlength=900).max() / a.N
    assert abs(share - w[0] / w.sum()) < 0.1 * w[0] / w.sum()
    # r = mu + signal + noise: signal variance ~1, noise 0.5^2
    assert abs(float(a.r.double().mean()) - 3.6) < 0.05
    assert abs(float(a.r.double().var()) - 1.25) < 0.1
    # the test set is a different stream of the same process
    assert not torch.equal(a.ut[:100], a.u[:100])


@pytest.mark.gpu
def test_cuda_rendering_is_bit_identical_to_cpu():
    if not torch.cuda.is_available():  # pragma: no cover
        pytest.skip("no CUDA device")
    for name, frac in (("netflix", 0.01), ("yahoo", 0.002), ("hugewiki", 0.0005)):
        c = synth.shaped(name, fraction=frac, device="cpu")
        g = synth.shaped(name, fraction=frac, device="cuda")
        assert synth.checksum(c) == synth.checksum(g), name
        assert torch.equal(c.r, g.r.cpu()) and torch.equal(c.v, g.v.cpu()), name


def test_table2_shapes_and_table3_hyperparameters():
    """Table 2 shapes and Table 3 hyper-parameters of the configs."""
    want = {"netflix": (480_190, 17_771, 99_072_112, 1_408_395, 0.05, 0.08, 0.3),
            "yahoo": (1_000_990, 624_961, 252_800_275, 4_003_960, 1.0, 0.08, 0.2),
            "hugewiki": (50_082_604, 39_781, 3_069_817_980, 31_327_899, 0.03, 0.08, 0.3)}
    for name, (m, n, N, Nt, lam, alpha, beta) in want.items():
        s = synth.SHAPES[name]
        assert (s["m"], s["n"], s["N"], s["Ntest"]) == (m, n, N, Nt), name
        assert (s["lam"], s["alpha"], s["beta"]) == (lam, alpha, beta), name
    R = synth.shaped("yahoo", fraction=0.0005)
    assert (R.m, R.n, R.N, R.Ntest) == (500, 312, 126_400, 2_001)
    assert 0.0 <= float(R.r.min()) and float(R.r.max()) <= 100.0      # Yahoo's 0-100 scale


def test_eq5_byte_and_flop_accounting():
    """Eq. 5: one update at k = 128 with fp32 features moves 12 + 4 k 4 = 2060 bytes
    for 7k - 1 = 895 flops, 0.43 flop/B -- the algorithmic bytes bench.py divides by (fp16: 1036)."""
    k = 128
    assert 12 + 4 * k * 4 == 2060 and 12 + 4 * k * 2 == 1036
    assert 7 * k - 1 == 895 and round(895 / 2060, 2) == 0.43
