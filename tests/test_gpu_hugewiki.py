"""configs[3] at full size on one B200: the Hugewiki-shaped set, N = 3,069,817,980 > 2^31 (and
m*k = 6.4e9 > 2^32), so every 64-bit index path of the library runs: the shuffle sort and the
slot placement over N, the init counter u*k + d, the chunk list, the RMSE grid-stride.
Properties that hold at any size, plus sampled outputs the oracle computes one by one (-m gpu)."""
import numpy as np
import pytest

from oracle import pyoracle as po
from paper_conf_hpdc_xietfl17_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_hpdc_xietfl17_b200 import mf  # noqa: E402

L = po.lib()
SEED = 42
HUGE = synth.SHAPES["hugewiki"]
HP = dict(lambda_p=HUGE["lam"], alpha=HUGE["alpha"], beta=HUGE["beta"])


def test_hugewiki_init_sampled_beyond_2_32():
    """P[u][d] = round_fp16((float)U24(S_P, u*k+d) * 2^-24 * sqrt(1/k)) at sampled rows, half of
    them with u*k + d >= 2^32 (the 64-bit init counter), and the last row."""
    m, n = HUGE["m"], HUGE["n"]
    u = torch.tensor([0, m - 1], dtype=torch.int32, device="cuda")
    v = torch.tensor([0, n - 1], dtype=torch.int32, device="cuda")
    r = torch.ones(2, dtype=torch.float32, device="cuda")
    g = mf.MF(m, n, 128, storage="fp16", seed=SEED, **HP)
    g.load(u, v, r)
    P, Q = g.factors(on_device=True)
    g.close()
    rng = np.random.default_rng(1)
    SP, SQ = L.or_stream(SEED, 4, 0, 0), L.or_stream(SEED, 5, 0, 0)
    amp = np.float32(np.sqrt(1.0 / 128))
    big = (1 << 32) // 128 + 1
    rows = [int(x) for x in rng.integers(0, m, 100)] + [int(x) for x in rng.integers(big, m, 100)]
    rows.append(m - 1)
    for X, S, idx in ((P, SP, rows), (Q, SQ, [int(x) for x in rng.integers(0, n, 100)])):
        for i in idx:
            d = int(rng.integers(128))
            u01 = np.float32(L.or_key(S, i * 128 + d) >> 40) * np.float32(2.0 ** -24)
            assert X[i, d].item() == L.or_round_storage(1, float(np.float32(u01 * amp))), (i, d)
    del P, Q
    torch.cuda.empty_cache()


def test_hugewiki_fullsize_hogwild_epoch():
    """The bench's --workload hugewiki configuration (fp16 Hogwild, k = 128, all resident
    workers): one epoch updates every one of the 3.07 B samples exactly once, and the test RMSE
    over the 31.3 M test ratings falls and stays finite."""
    R = synth.shaped("hugewiki", device="cuda")
    assert R.N == HUGE["N"] and R.N > 2 ** 31
    g = mf.MF(R.m, R.n, 128, storage="fp16", seed=SEED, **HP)
    g.load(R.u, R.v, R.r)
    g.load(R.ut, R.vt, R.rt, "test")
    N = R.N
    del R
    torch.cuda.empty_cache()
    r0 = g.rmse()
    g.train_epoch()
    st = g.stats()
    cv = g.check_visits()
    r1 = g.rmse()
    g.close()
    assert st["updates"] == N and st["sgd_launches"] == 1      # device count, N > 2^31
    assert cv["bad_units"] == 0 and cv["units"] == -(-N // 256), cv   # 11,991,477 chunks once
    assert np.isfinite(r1) and r1 < r0, (r0, r1)


def test_yahoo_fullsize_wavefront_bit_identical_rerun():
    """configs[2] at full size (252.8 M ratings, 1.0 M x 625 K): the deterministic wavefront in
    its swept configuration (fp32, s = 888, c = 15360, cyclic) gives bit-identical factors on a
    rerun (a property of the serial (w, i) order at any size), and lowers the test RMSE."""
    Y = synth.SHAPES["yahoo"]
    R = synth.shaped("yahoo", device="cuda")
    hp = dict(lambda_p=Y["lam"], alpha=Y["alpha"], beta=Y["beta"], rating_scale=Y["rating_scale"])
    outs = []
    for _ in range(2):
        g = mf.MF(R.m, R.n, 128, storage="fp32", schedule="wavefront", workers=888, wf_cols=15360,
                  cyclic=True, seed=SEED, **hp)
        g.load(R.u, R.v, R.r)
        g.load(R.ut, R.vt, R.rt, "test")
        r0 = g.rmse()
        g.train_epoch()
        r1 = g.rmse()
        assert g.stats()["updates"] == R.N and r1 < r0, (r0, r1)
        outs.append(g.factors(on_device=True))
        g.close()
    assert torch.equal(outs[0][0], outs[1][0]) and torch.equal(outs[0][1], outs[1][1])
