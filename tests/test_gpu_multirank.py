"""The world > 1 GPU path (DSGD strata, Q-segment rotation, row-filtered test RMSE with an
all-reduce, factor gathering) on ONE GPU through the loopback transport (-m gpu): ranks are
ctxs of this process, one host thread each, exchanging Q segments by device-to-device copies.
The plan and protocol are the NCCL path's.  Blocks of a stratum touch disjoint P/Q rows, so
the result equals the oracle's serial strata loop (grid a = 8) for any world size.
"""
import os
import threading

import numpy as np
import pytest

from oracle import pyoracle as po
from paper_conf_hpdc_xietfl17_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_hpdc_xietfl17_b200 import mf  # noqa: E402

HP = dict(lambda_p=0.05, alpha=0.08, beta=0.3, seed=77)


def run_ranks(world, R, k, epochs, **kw):
    key = os.urandom(16).ljust(128, b"\0")
    out = [None] * world
    errs = []

    def work(rank):
        try:
            m = mf.MF(R.m, R.n, k, world=world, rank=rank, transport=1, nccl_id=key, grid_a=8,
                      **HP, **kw)
            m.load(R.u, R.v, R.r)
            m.load(R.ut, R.vt, R.rt, "test")
            for _ in range(epochs):
                m.train_epoch()
            rm = m.rmse()
            P, Q = m.factors()
            out[rank] = (rm, P, Q, m.stats(), m.check_visits())
            m.close()
        except Exception as e:  # surface in the main thread
            errs.append(e)

    th = [threading.Thread(target=work, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not any(t.is_alive() for t in th), "a rank hung"
    if errs:
        raise errs[0]
    return out


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("kw", [dict(schedule="wavefront", workers=4, wf_cols=5),
                                dict(schedule="hogwild", workers=1, batch_f=64),
                                dict(schedule="wavefront", workers=4, wf_cols=5, staged=True),
                                dict(schedule="hogwild", workers=1, batch_f=64, group_cols=True)])
def test_multirank_strata_matches_oracle(world, kw):
    R = synth.tiny(seed=0)
    epochs = 2
    res = run_ranks(world, R, 16, epochs, **kw)
    okw = {k: v for k, v in kw.items() if k != "staged"}
    o = po.Oracle(R.m, R.n, 16, R.u, R.v, R.r, grid_a=8, **HP, **okw)
    for _ in range(epochs):
        o.train_epoch()
    Po, Qo = o.factors()
    ro = o.rmse(R.ut, R.vt, R.rt)
    for rank, (rm, P, Q, st, cv) in enumerate(res):
        assert cv["bad_units"] == 0 and cv["epochs"] == epochs, (rank, cv)
        assert np.array_equal(P, res[0][1]) and np.array_equal(Q, res[0][2]), rank
        assert rm == res[0][0]
        assert np.abs(P - Po).max() <= 2e-4 and np.abs(Q - Qo).max() <= 2e-4
        assert abs(rm - ro) <= 2e-5 * ro, (rm, ro)
    # every rank trained only its own blocks: the device-counted updates add up to N per epoch
    assert sum(r[3]["updates"] for r in res) == R.N


def test_multirank_equals_single_gpu_strata():
    """world 2 vs world 1 with the same a = 8 grid: identical schedule -> identical factors
    (deterministic wavefront; both are the same sequence of block runs)."""
    R = synth.uniform(m=500, n=300, N=30_000, seed=3, mu=1.0, rank=3, noise=0.1, Ntest=3000)
    kw = dict(schedule="wavefront", workers=4, wf_cols=6)
    two = run_ranks(2, R, 32, 2, **kw)
    one = mf.MF(R.m, R.n, 32, grid_a=8, **HP, **kw)
    one.load(R.u, R.v, R.r)
    one.load(R.ut, R.vt, R.rt, "test")
    for _ in range(2):
        one.train_epoch()
    P1, Q1 = one.factors()
    assert np.array_equal(two[0][1], P1) and np.array_equal(two[0][2], Q1)
    assert abs(two[0][0] - one.rmse()) <= 1e-12 * one.rmse() + 1e-15
