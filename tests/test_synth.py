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
