"""Multi-process DSGD-strata protocol on CPU (gloo, world_size 2 and 4; -m "not gpu").

Every rank runs the plan produced by the product's host planner mf_strata_plan (the very
function mf_train_epoch executes before each sub-epoch): it trains the strata blocks of its
own row segments with the CPU oracle, and moves the Q segments the plan lists (relabelled
column-row ranges) between processes with gloo isend/irecv.  Because the blocks of a stratum
touch disjoint rows of P and Q, the distributed result must equal the single-process oracle's
serial strata loop (A: "Oracle serialization of an epoch") BIT-EXACTLY: owned P rows on every
rank, and every Q segment on its final holder.  This checks the planner's block assignment,
holder tracking across sub-epochs and epochs, and segment ranges; the GPU path replaces the
oracle with the SGD kernels and gloo with NCCL.
"""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import pyoracle as po
from paper_conf_hpdc_xietfl17_b200 import build, mf, synth

SEED = 4242
A = 8
EPOCHS = 2
K = 4


def _data():
    return synth.uniform(m=97, n=61, N=4000, seed=11, mu=1.0, rank=2, noise=0.1)


def _oracle(R, kw):
    return po.Oracle(R.m, R.n, K, R.u, R.v, R.r, seed=SEED, grid_a=A, lambda_p=0.05, alpha=0.08,
                     beta=0.3, **kw)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, kw, outdir):
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        R = _data()
        o = _oracle(R, kw)
        rho_c = o.export("rho_c")
        holders = [-1] * A
        for t in range(EPOCHS):
            for j in range(A):
                blocks, xfers, holders = mf.strata_plan(SEED, A, world, rank, R.n, t, j, holders)
                reqs, recvs = [], []
                _, Q = o.factors()
                for (J, src, dst, lo, hi) in xfers:
                    cols = np.nonzero((rho_c >= lo) & (rho_c < hi))[0]
                    if src == rank:
                        reqs.append(dist.isend(torch.from_numpy(np.ascontiguousarray(Q[cols])),
                                               dst, tag=int(J)))
                    if dst == rank:
                        buf = torch.empty((len(cols), K), dtype=torch.float32)
                        reqs.append(dist.irecv(buf, src, tag=int(J)))
                        recvs.append((cols, buf))
                for r in reqs:
                    r.wait()
                if recvs:
                    for cols, buf in recvs:
                        Q[cols] = buf.numpy()
                    o.set_factors(Q=Q)
                for b in blocks:
                    o.run_block(t, int(b))
        P, Q = o.factors()
        np.savez(os.path.join(outdir, f"rank{rank}.npz"), P=P, Q=Q, holders=np.array(holders))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("kw", [dict(schedule="hogwild", batch_f=32),
                                dict(schedule="wavefront", workers=3, wf_cols=4)])
def test_distributed_strata_equals_serial_oracle(world, kw):
    build.build()
    R = _data()
    ref = _oracle(R, kw)
    for _ in range(EPOCHS):
        ref.train_epoch()
    Pr, Qr = ref.factors()
    rho_r, rho_c = ref.export("rho_r"), ref.export("rho_c")
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(world, _free_port(), kw, d), nprocs=world, join=True)
        res = [np.load(os.path.join(d, f"rank{g}.npz")) for g in range(world)]
    per = A // world
    seg_r = rho_r * A // R.m
    seg_c = rho_c * A // R.n
    holders = res[0]["holders"]
    for g in range(world):
        assert np.array_equal(res[g]["holders"], holders)       # every rank tracks the same plan
        own = (seg_r >= g * per) & (seg_r < (g + 1) * per)
        assert own.any()
        assert np.array_equal(res[g]["P"][own], Pr[own]), f"P rows of rank {g}"
    for J in range(A):
        h = int(holders[J])
        sel = seg_c == J
        assert np.array_equal(res[h]["Q"][sel], Qr[sel]), f"Q segment {J} on rank {h}"
    # the run trained something: factors moved away from the initial values
    P0, _ = _oracle(R, kw).factors()
    assert not np.array_equal(Pr, P0)


def test_plan_covers_each_stratum_once():
    """Union over ranks of the planned blocks in sub-epoch j = the stratum {(r, (r+pi_t[j]) mod a)};
    each rank trains only its own row segments; transfers only leave the current holder."""
    build.build()
    o = po.Oracle(64, 64, 2, [0], [0], [1.0], seed=SEED, grid_a=A)
    for world in (1, 2, 4, 8):
        hold = {g: [-1] * A for g in range(world)}
        for t in range(3):
            pi = o.export("strata", t)
            for j in range(A):
                got = []
                for g in range(world):
                    blocks, xf, hold[g] = mf.strata_plan(SEED, A, world, g, 64, t, j, hold[g])
                    for b in blocks:
                        assert (b // A) // (A // world) == g
                    for (J, src, dst, lo, hi) in xf:
                        assert src != dst and 0 <= lo < hi <= 64
                    got += blocks
                assert sorted(got) == sorted(r * A + (r + pi[j]) % A for r in range(A))
                assert all(hold[g] == hold[0] for g in range(world))
