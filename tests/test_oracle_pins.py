"""Pins of the CPU oracle against things other than itself (-m "not gpu").

Each test names what fixes the expected value: a published constant, a hand-worked example,
a closed form, an independent library routine (numpy / torch conversions), or brute force.
"""
import itertools
import json
import math
import os

import numpy as np
import pytest
import torch

from oracle import pyoracle as po

L = po.lib()
PHI = 0x9E3779B97F4A7C15


def golden(golden_dir, name):
    with open(os.path.join(golden_dir, name)) as f:
        return json.load(f)


# --------------------------------------------------------------------------- hashing (App. A)

def test_mix_is_published_splitmix64(golden_dir):
    """mix = SplitMix64 finaliser: key(0, i) = mix(i*phi) is the i-th SplitMix64 output from
    state 0, whose first values are published with the reference implementation."""
    g = golden(golden_dir, "appendix_a.json")
    got = [L.or_key(0, i) for i in range(1, 5)]
    assert got == [int(x, 16) for x in g["splitmix64_seed0_first4"]]


def test_appendix_a_golden_vectors(golden_dir):
    """SURVEY App. A golden vectors (independent Python rendering of the spec, seed 42)."""
    g = golden(golden_dir, "appendix_a.json")
    s = g["seed"]
    S = L.or_stream(s, 1, 0, 0)
    assert S == int(g["S_SHUF"], 16)
    assert [L.or_key(S, i) for i in range(3)] == [int(x, 16) for x in g["key_S_SHUF_0_2"]]
    assert po.perm(S, 10).tolist() == g["perm_S_SHUF_10"]
    pr = po.perm(L.or_stream(s, 2, 0, 0), 10)
    assert pr.tolist() == g["perm_S_ROW_10"]
    assert po.perm(L.or_stream(s, 6, 0, 0), 8).tolist() == g["perm_S_HW_0_0_8"]
    for i, want in enumerate(g["perm_S_WF_0_0_i_8"]):
        assert po.perm(L.or_stream(s, 7, 0, i), 8).tolist() == want
    assert po.perm(L.or_stream(s, 8, 0, 0), 8).tolist() == g["pi_0_a8"]
    # the same values through a whole oracle context (relabel, strata order, init)
    m = 10
    o = po.Oracle(m, 10, 16, [0], [0], [1.0], seed=s, grid_a=8)
    assert o.export("rho_r").tolist() == g["rho_R_10"]
    assert o.export("strata", 0).tolist() == g["pi_0_a8"]
    P, _ = o.factors()
    np.testing.assert_allclose(P[0, :4], g["init_k16_P0_0_3_fp32"], rtol=2e-7)
    o16 = po.Oracle(m, 10, 16, [0], [0], [1.0], seed=s, storage="fp16")
    P16, _ = o16.factors()
    np.testing.assert_allclose(P16[0, :4], g["init_k16_P0_0_3_fp16"], rtol=5e-4)


def test_ctx_storage_order_is_perm_S_SHUF(golden_dir):
    """Alg. 1 l.2 random_shuffle through a whole context: the storage order of an N = 10
    training set is perm(S_SHUF, 10) of App. A's golden vectors (caller index per position)."""
    g = golden(golden_dir, "appendix_a.json")
    u = np.arange(10, dtype=np.int32)
    o = po.Oracle(10, 10, 16, u, u[::-1].copy(), np.ones(10, np.float32), seed=g["seed"])
    assert o.export("perm").tolist() == g["perm_S_SHUF_10"]
    ow = po.Oracle(10, 10, 16, u, u[::-1].copy(), np.ones(10, np.float32), seed=g["seed"],
                   schedule="wavefront", workers=2, wf_cols=3)
    assert ow.export("perm").tolist() == g["perm_S_SHUF_10"]


def _grid_case(golden_dir, **kw):
    g = golden(golden_dir, "appendix_a_blocks.json")
    cs = g["case"]
    u = np.repeat(np.arange(cs["m"], dtype=np.int32), cs["n"])
    v = np.tile(np.arange(cs["n"], dtype=np.int32), cs["m"])
    r = np.ones(cs["N"], np.float32)
    o = po.Oracle(cs["m"], cs["n"], 16, u, v, r, seed=42, grid_a=cs["a"], **kw)
    return g, cs, o


def test_block_and_subblock_ids_hand_derived(golden_dir):
    """App. A 'Segments and blocks' on m = 10, n = 7 (ragged column segments 4 + 3), a = 2,
    s = 3, c = 4: relabel ranks, strata block and wavefront sub-block of every cell against the
    hand derivation in tests/golden/appendix_a_blocks.json (segment-LOCAL sub-block index with
    ceil segment starts: using m instead of m_r, or floor starts, changes several ids)."""
    g, cs, o = _grid_case(golden_dir, schedule="wavefront", workers=3, wf_cols=4)
    assert o.export("rho_r").tolist() == g["rho_R"]
    assert o.export("rho_c").tolist() == g["rho_C"]
    perm = o.export("perm")
    blk = np.empty(cs["N"], np.int64)
    blk[perm] = o.export("blockid")                     # by caller index i = 7u + v
    assert blk.reshape(cs["m"], cs["n"]).tolist() == g["wavefront_blockid_by_u_v"]
    _, _, oh = _grid_case(golden_dir, schedule="hogwild")
    hb = np.empty(cs["N"], np.int64)
    hb[oh.export("perm")] = oh.export("blockid")
    assert hb.reshape(cs["m"], cs["n"]).tolist() == g["hogwild_blockid_by_u_v"]


def test_cyclic_sequences_and_tickets_hand_derived(golden_dir):
    """App. A cyclic variant: seq_i[w] = sigma[(tau[i] + w) mod c] per strata block, and the
    (w, i)-lexicographic ticket ranks, against values derived by hand from tau and sigma."""
    g, cs, o = _grid_case(golden_dir, schedule="wavefront", workers=3, wf_cols=4, cyclic=True)
    for b in range(4):
        tau, sigma = g["cyclic_tau_sigma_t0"][f"b{b}"]
        assert po.perm(L.or_stream(42, 9, 0, b), 4).tolist() == tau
        assert po.perm(L.or_stream(42, 10, 0, b), 4).tolist() == sigma
    seq = o.export("wfseq", 0).reshape(12, 4).tolist()
    assert seq == g["cyclic_wfseq_t0"]
    assert o.export("tickets", 0).reshape(12, 4).tolist() == g["cyclic_tickets_t0"]
    # the epoch's execution order: strata pi_0 = [0, 1] for a = 2 -> blocks 0, 3, 1, 2; in each,
    # for w: for i: sub-block (i, seq_i[w]) in storage order
    assert o.export("strata", 0).tolist() == [0, 1]
    sub = o.export("blockid")                            # per storage position
    want = []
    for b in (0, 3, 1, 2):
        for w in range(4):
            for i in range(3):
                sb = (b * 3 + i) * 4 + g["cyclic_wfseq_t0"][b * 3 + i][w]
                want += [j for j in range(cs["N"]) if sub[j] == sb]
    assert o.export("order", 0).tolist() == want


def test_keys_distinct_and_perm_is_sorted_permutation():
    S = L.or_stream(7, 1, 0, 0)
    n = 200_000
    p = po.perm(S, n)
    assert np.array_equal(np.sort(p), np.arange(n))
    keys = np.array([L.or_key(S, int(i)) for i in p[:2000]], dtype=np.uint64)
    assert np.all(keys[1:] > keys[:-1])


# --------------------------------------------------------------------------- storage rounding

def _probe_floats(n=400_000, seed=0):
    rng = np.random.default_rng(seed)
    mant = rng.integers(0, 1 << 23, n, dtype=np.uint32)
    expo = rng.integers(127 - 30, 127 + 17, n, dtype=np.uint32)  # spans subnormal..overflow
    sign = rng.integers(0, 2, n, dtype=np.uint32) << 31
    x = (sign | (expo << 23) | mant).view(np.float32)
    # exact halfway cases of fp16 normals and subnormals, and the overflow boundary
    half_ties = (np.arange(1, 2000, dtype=np.float32) + 0.5) * np.float32(2.0 ** -24)
    extra = np.array([0.0, -0.0, 65504.0, 65519.99, 65520.0, 2.0 ** -25, 2.0 ** -25 * 1.0000001,
                      2.0 ** -24, 6.1035156e-05, 1.0 + 2.0 ** -11, 1.0 + 3 * 2.0 ** -11],
                     dtype=np.float32)
    return np.concatenate([x, half_ties, -half_ties, extra])


def test_f16_encoder_matches_numpy_ieee_rne():
    """The oracle's software binary16 encoder vs numpy's IEEE round-to-nearest-even cast."""
    x = _probe_floats()
    with np.errstate(over="ignore"):
        want = x.astype(np.float16).view(np.uint16)
    got = np.array([L.or_f16_bits(float(v)) for v in x], dtype=np.uint16)
    bad = np.nonzero(got != want)[0]
    assert bad.size == 0, (x[bad[:5]], got[bad[:5]], want[bad[:5]])
    back = np.array([L.or_f16_value(int(h)) for h in want[:20000]], dtype=np.float32)
    np.testing.assert_array_equal(back, want[:20000].view(np.float16).astype(np.float32))


def test_bf16_encoder_matches_torch_rne():
    x = _probe_floats(200_000, seed=1)
    x = x[np.abs(x) < 1e30]
    want = torch.from_numpy(x).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    got = np.array([L.or_bf16_bits(float(v)) for v in x], dtype=np.uint16)
    assert np.array_equal(got, want)


# --------------------------------------------------------------------------- one update

def test_hand_update_dyadic_exact(golden_dir):
    """Alg. 1 l.8-10 by hand (dyadic: exact in fp32 and fp16)."""
    h = golden(golden_dir, "hand_update.json")["dyadic"]
    for storage in ("fp32", "fp16", "bf16"):
        p, q = po.update(h["p"], h["q"], h["r"], h["gamma"], h["lambda"], h["lambda"], storage)
        assert p.tolist() == h["p_new"]
        assert q.tolist() == h["q_new"]
        assert q.tolist() != h["q_new_if_sequential_reading"]


def test_hand_update_nondyadic(golden_dir):
    h = golden(golden_dir, "hand_update.json")["nondyadic"]
    p, q = po.update(h["p"], h["q"], h["r"], h["gamma"], h["lambda"], h["lambda"])
    np.testing.assert_allclose(p, h["p_new"], atol=h["tol"])
    np.testing.assert_allclose(q, h["q_new"], atol=h["tol"])


def test_update_is_half_gradient_step_of_eq3():
    """Central finite differences of Eq. 3 equal 2(p - p')/gamma (R2): the update is a
    gradient step with gamma absorbing the factor 2.  Fails for a dropped term, a wrong sign,
    a swapped p/q, or the sequential reading of line 10."""
    rng = np.random.default_rng(3)
    for trial in range(20):
        k = int(rng.choice([1, 2, 7, 16]))
        p = rng.normal(size=k).astype(np.float32)
        q = rng.normal(size=k).astype(np.float32)
        r = float(rng.normal() * 2)
        lp, lq = float(rng.uniform(0, 1)), float(rng.uniform(0, 1))
        g = 0.05
        p1, q1 = po.update(p, q, r, g, lp, lq)
        h = 1e-6
        gp = np.zeros(k)
        gq = np.zeros(k)
        pd, qd = p.astype(np.float64), q.astype(np.float64)
        for d in range(k):
            e = np.zeros(k); e[d] = h
            gp[d] = (po.sample_loss(pd + e, qd, r, lp, lq) - po.sample_loss(pd - e, qd, r, lp, lq)) / (2 * h)
            gq[d] = (po.sample_loss(pd, qd + e, r, lp, lq) - po.sample_loss(pd, qd - e, r, lp, lq)) / (2 * h)
        step_p = 2 * (pd - p1.astype(np.float64)) / g
        step_q = 2 * (qd - q1.astype(np.float64)) / g
        np.testing.assert_allclose(step_p, gp, rtol=2e-3, atol=2e-3)
        np.testing.assert_allclose(step_q, gq, rtol=2e-3, atol=2e-3)


def test_update_special_cases():
    rng = np.random.default_rng(4)
    p = rng.normal(size=16).astype(np.float32)
    q = rng.normal(size=16).astype(np.float32)
    # gamma = 0: nothing moves
    p1, q1 = po.update(p, q, 3.0, 0.0, 0.3, 0.3)
    assert np.array_equal(p1, p) and np.array_equal(q1, q)
    # lambda = 0 and r = p.q exactly: fixed point (dyadic values so the dot is exact)
    pe = np.array([0.5, -1.25, 2.0], dtype=np.float32)
    qe = np.array([1.5, 0.25, -0.75], dtype=np.float32)
    r = float(np.dot(pe.astype(np.float64), qe))
    p1, q1 = po.update(pe, qe, r, 0.1, 0.0, 0.0)
    assert np.array_equal(p1, pe) and np.array_equal(q1, qe)
    # k = 1, lambda = 0: e' = e (1 - g (p^2 + q^2) - g^2 e p q)   (closed form, in double)
    pp, qq, rr, g = 0.7, -0.4, 1.3, 0.05
    e = rr - pp * qq
    p1, q1 = po.update([pp], [qq], rr, g, 0.0, 0.0)
    e_new = rr - float(p1[0]) * float(q1[0])
    assert abs(e_new - e * (1 - g * (pp * pp + qq * qq) - g * g * e * pp * qq)) < 1e-6
    # ... and repeating it converges p.q -> r geometrically
    P, Q = np.float32([pp]), np.float32([qq])
    for _ in range(400):
        P, Q = po.update(P, Q, rr, g, 0.0, 0.0)
    assert abs(rr - float(P[0]) * float(Q[0])) < 1e-5


def test_gamma_schedule_closed_form():
    """Eq. 9 at t = 0 (gamma_0 = alpha, R4) and at perfect squares, where t^1.5 is an
    integer; plus Table 3 Netflix values (alpha .08, beta .3)."""
    for a, b in [(0.08, 0.3), (0.08, 0.2), (0.05, 0.0), (1.0, 1.0)]:
        a32, b32 = float(np.float32(a)), float(np.float32(b))
        assert L.or_gamma(a, b, 0) == np.float32(a)
        for t, t15 in [(1, 1), (4, 8), (9, 27), (16, 64), (100, 1000)]:
            assert L.or_gamma(a, b, t) == np.float32(a32 / (1 + b32 * t15))
    want = [0.08, 0.06153846, 0.043277673, 0.031264096]
    got = [L.or_gamma(0.08, 0.3, t) for t in range(4)]
    np.testing.assert_allclose(got, want, rtol=1e-7)
    assert all(x > y for x, y in zip(got, got[1:]))


# --------------------------------------------------------------------------- schedules

def _tiny_uniform(m=60, n=50, N=3000, seed=5):
    rng = np.random.default_rng(seed)
    return (rng.integers(0, m, N).astype(np.int32), rng.integers(0, n, N).astype(np.int32),
            rng.normal(size=N).astype(np.float32), m, n)


SCHEDULES = [
    dict(schedule="hogwild", batch_f=7),
    dict(schedule="hogwild", batch_f=256),
    dict(schedule="wavefront", workers=4, wf_cols=8),
    dict(schedule="wavefront", workers=3, wf_cols=5),
    dict(schedule="wavefront", workers=4, wf_cols=8, cyclic=True),
    dict(schedule="hogwild", batch_f=16, grid_a=8),
    dict(schedule="wavefront", workers=2, wf_cols=3, grid_a=4),
]


@pytest.mark.parametrize("kw", SCHEDULES)
def test_every_sample_exactly_once_per_epoch(kw):
    u, v, r, m, n = _tiny_uniform()
    o = po.Oracle(m, n, 4, u, v, r, **kw)
    for t in range(3):
        order = o.export("order", t)
        assert np.array_equal(np.sort(order), np.arange(len(u)))


def test_serial_special_cases_reduce_to_algorithm_1():
    """s = c = a = 1 wavefront and f >= N Hogwild both run the storage order verbatim
    (Alg. 1: one shuffled pass)."""
    u, v, r, m, n = _tiny_uniform()
    for kw in (dict(schedule="wavefront", workers=1, wf_cols=1),
               dict(schedule="hogwild", batch_f=1 << 20)):
        o = po.Oracle(m, n, 4, u, v, r, **kw)
        assert np.array_equal(o.export("order", 0), np.arange(len(u)))
    # and training in that order equals the update applied by hand in storage order
    o = po.Oracle(m, n, 4, u, v, r, schedule="wavefront", workers=1, wf_cols=1, seed=9)
    P, Q = o.factors()
    perm = o.export("perm")
    g = L.or_gamma(0.08, 0.3, 0)
    for i in perm:
        P[u[i]], Q[v[i]] = po.update(P[u[i]], Q[v[i]], float(r[i]), g, 0.05, 0.05)
    o.train_epoch()
    P2, Q2 = o.factors()
    assert np.array_equal(P, P2) and np.array_equal(Q, Q2)


def test_hogwild_chunks_are_consecutive_storage_runs():
    u, v, r, m, n = _tiny_uniform()
    f = 64
    o = po.Oracle(m, n, 4, u, v, r, schedule="hogwild", batch_f=f)
    order = o.export("order", 1)
    co = o.export("chunkorder", 1)
    assert np.array_equal(np.sort(co), np.arange(len(co)))
    want = np.concatenate([np.arange(c * f, min((c + 1) * f, len(u))) for c in co])
    assert np.array_equal(order, want)
    # a permutation of chunks that changes with the epoch
    assert not np.array_equal(co, o.export("chunkorder", 0))


def test_wavefront_tickets_brute_force_and_fig6_golden(golden_dir):
    """Ticket rank of (w,i) = #earlier visits (lexicographic (w,i)) of the same column.
    Golden: seed 42, s=4, c=8: workers 0, 1, 3 all start at column 0 -> tickets 0, 1, 2
    (the Fig. 6 narrative P:L287-289 of a worker waiting for a column)."""
    g = golden(golden_dir, "appendix_a.json")
    s, c = 4, 8
    o = po.Oracle(20, 20, 2, [0], [0], [1.0], seed=42, schedule="wavefront", workers=s, wf_cols=c)
    seq = o.export("wfseq", 0).reshape(s, c)
    assert seq.tolist() == g["perm_S_WF_0_0_i_8"]
    tk = o.export("tickets", 0).reshape(s, c)
    assert [tk[0, 0], tk[1, 0], tk[3, 0]] == [0, 1, 2]
    for i in range(s):
        for w in range(c):
            col = seq[i, w]
            cnt = sum(1 for w2 in range(c) for i2 in range(s)
                      if (w2, i2) < (w, i) and seq[i2, w2] == col)
            assert tk[i, w] == cnt
    # every column is visited exactly s times per epoch: ranks 0..s-1 per column
    for col in range(c):
        assert sorted(tk[seq == col].tolist()) == list(range(s))


def test_wavefront_cyclic_has_no_same_wave_column_conflicts():
    s, c = 5, 9
    o = po.Oracle(30, 30, 2, [0], [0], [1.0], schedule="wavefront", workers=s, wf_cols=c,
                  cyclic=True)
    seq = o.export("wfseq", 3).reshape(s, c)
    for i in range(s):
        assert sorted(seq[i].tolist()) == list(range(c))
    for w in range(c):
        assert len(set(seq[:, w].tolist())) == s


def test_wavefront_blocks_respect_eq6_within_a_wave_order():
    """Replaying the oracle's order, two updates of the same row sub-block or column sub-block
    never interleave across different blocks: each (i,j) block runs contiguously, and a
    worker's blocks appear in its wave order."""
    u, v, r, m, n = _tiny_uniform(N=4000)
    s, c = 4, 8
    o = po.Oracle(m, n, 4, u, v, r, schedule="wavefront", workers=s, wf_cols=c)
    blk = o.export("blockid", 0)
    order = o.export("order", 0)
    seq = o.export("wfseq", 0).reshape(s, c)
    runs = [blk[order[0]]]
    for j in order[1:]:
        if blk[j] != runs[-1]:
            runs.append(blk[j])
    assert len(runs) == len(set(runs))          # each block is one contiguous run
    pos = {b: x for x, b in enumerate(runs)}
    for i in range(s):
        ids = [i * c + seq[i, w] for w in range(c) if (i * c + seq[i, w]) in pos]
        assert [pos[b] for b in ids] == sorted(pos[b] for b in ids)


def test_block_assignment_segments_are_balanced_and_consistent():
    u, v, r, m, n = _tiny_uniform(m=97, n=61, N=5000)
    a = 8
    o = po.Oracle(m, n, 4, u, v, r, grid_a=a)
    rho_r, rho_c = o.export("rho_r"), o.export("rho_c")
    assert np.array_equal(np.sort(rho_r), np.arange(m))
    assert np.array_equal(np.sort(rho_c), np.arange(n))
    seg_r = rho_r * a // m
    sizes = np.bincount(seg_r, minlength=a)
    assert sizes.max() - sizes.min() <= 1
    # (the block ids themselves are pinned by hand-derived values in
    # test_block_and_subblock_ids_hand_derived)


def _feasible_orders_2x2():
    """Fig. 15: 2x2 blocks, 2 workers; an order b1 b2 b3 b4 is feasible iff the
    concurrently running pairs (b1,b2) and (b3,b4) are independent (Eq. 6 at block level)."""
    rc = {1: (0, 0), 2: (0, 1), 3: (1, 0), 4: (1, 1)}

    def indep(x, y):
        return rc[x][0] != rc[y][0] and rc[x][1] != rc[y][1]

    return [o for o in itertools.permutations([1, 2, 3, 4]) if indep(o[0], o[1]) and indep(o[2], o[3])]


def test_fig15_feasible_block_orders_and_strata_order():
    feas = _feasible_orders_2x2()
    assert len(feas) == 8 and len(list(itertools.permutations(range(4)))) == 24
    # the strata order with a = 2 run by 2 workers is always one of the feasible orders,
    # and every stratum's a blocks are pairwise independent for a = 8
    u, v, r, m, n = _tiny_uniform()
    o2 = po.Oracle(m, n, 2, u, v, r, grid_a=2)
    for t in range(6):
        pi = o2.export("strata", t)
        order = tuple(1 + rr * 2 + (rr + pi[j]) % 2 for j in range(2) for rr in range(2))
        assert order in feas
    o8 = po.Oracle(m, n, 2, u, v, r, grid_a=8)
    for t in range(3):
        pi = o8.export("strata", t)
        assert sorted(pi.tolist()) == list(range(8))
        for j in range(8):
            cols = [(rr + pi[j]) % 8 for rr in range(8)]
            assert len(set(cols)) == 8


def test_run_block_in_strata_order_equals_train_epoch():
    u, v, r, m, n = _tiny_uniform()
    kw = dict(schedule="wavefront", workers=2, wf_cols=3, grid_a=4, seed=11)
    a = 4
    o1 = po.Oracle(m, n, 4, u, v, r, **kw)
    o2 = po.Oracle(m, n, 4, u, v, r, **kw)
    for t in range(2):
        o1.train_epoch()
        pi = o2.export("strata", t)
        for j in range(a):
            for rr in range(a):
                o2.run_block(t, rr * a + (rr + pi[j]) % a)
    o2.set_epoch(2)
    assert np.array_equal(o1.factors()[0], o2.factors()[0])
    assert np.array_equal(o1.factors()[1], o2.factors()[1])


# --------------------------------------------------------------------------- training

def _tiny_set():
    from paper_conf_hpdc_xietfl17_b200 import synth
    return synth.tiny(seed=0)


def test_init_distribution():
    """Alg. 1 l.3: U[0, a), a = sqrt(1/(k*scale)) (R5)."""
    k = 16
    o = po.Oracle(1000, 800, k, [0], [0], [0.0], init_scale=1.0)
    P, Q = o.factors()
    a = math.sqrt(1 / k)
    for X in (P, Q):
        assert X.min() >= 0 and X.max() < a
        assert abs(X.mean() - a / 2) < 0.01 * a
    o2 = po.Oracle(1000, 800, k, [0], [0], [0.0], init_scale=4.0)
    assert o2.factors()[0].max() < math.sqrt(1 / (4 * k))


def test_rmse_textbook_and_closed_forms():
    R = _tiny_set()
    o = po.Oracle(R.m, R.n, 16, R.u, R.v, R.r)
    o.train_epoch()
    P, Q = o.factors()
    pred = np.einsum("ij,ij->i", P[R.ut].astype(np.float64), Q[R.vt].astype(np.float64))
    want = np.sqrt(np.mean((R.rt.astype(np.float64) - pred) ** 2))
    assert abs(o.rmse(R.ut, R.vt, R.rt) - want) < 1e-5 * want
    # P = 0: prediction 0, RMSE = sqrt(mean r^2); rating_scale multiplies back
    o.set_factors(P=np.zeros_like(P))
    assert abs(o.rmse(R.ut, R.vt, R.rt) - np.sqrt(np.mean(R.rt.astype(np.float64) ** 2))) < 1e-6
    o4 = po.Oracle(R.m, R.n, 16, R.u, R.v, R.r, rating_scale=4.0)
    o4.set_factors(P=np.zeros_like(P))
    assert abs(o4.rmse(R.ut, R.vt, R.rt) - np.sqrt(np.mean(R.rt.astype(np.float64) ** 2))) < 1e-5


def test_loss_is_eq2_sum():
    R = _tiny_set()
    o = po.Oracle(R.m, R.n, 16, R.u[:500], R.v[:500], R.r[:500], lambda_p=0.1, lambda_q=0.2)
    P, Q = o.factors()
    p, q = P[R.u[:500]].astype(np.float64), Q[R.v[:500]].astype(np.float64)
    e = R.r[:500].astype(np.float64) - (p * q).sum(1)
    lp, lq = float(np.float32(0.1)), float(np.float32(0.2))  # the oracle holds lambda as float
    want = (e ** 2 + lp * (p ** 2).sum(1) + lq * (q ** 2).sum(1)).sum()
    assert abs(o.loss() - want) < 1e-9 * want


@pytest.mark.parametrize("schedule", ["hogwild", "wavefront"])
def test_training_loss_monotone_table3_netflix(schedule):
    """Eq. 2 decreases every epoch on tiny with Table 3 Netflix parameters."""
    R = _tiny_set()
    kw = dict(workers=8, wf_cols=16) if schedule == "wavefront" else {}
    o = po.Oracle(R.m, R.n, 16, R.u, R.v, R.r, lambda_p=0.05, alpha=0.08, beta=0.3,
                  schedule=schedule, **kw)
    losses = [o.loss()]
    for _ in range(10):
        o.train_epoch()
        losses.append(o.loss())
    assert all(b < a for a, b in zip(losses, losses[1:])), losses


def test_planted_recovery():
    """Planted rank-4 noiseless tiny set: SGD recovers it (SURVEY 8(c) calibration)."""
    R = _tiny_set()
    std = float(np.std(R.r))
    o = po.Oracle(R.m, R.n, 16, R.u, R.v, R.r, lambda_p=0.05, alpha=0.08, beta=0.3)
    for _ in range(10):
        o.train_epoch()
    assert o.rmse(R.ut, R.vt, R.rt) <= 0.30 * std
    o = po.Oracle(R.m, R.n, 16, R.u, R.v, R.r, lambda_p=0.0, alpha=0.05, beta=0.0)
    for _ in range(40):
        o.train_epoch()
    assert o.rmse(R.ut, R.vt, R.rt) <= 0.10 * std
    assert o.rmse(R.u, R.v, R.r) <= 0.03 * std


def test_fp16_storage_keeps_values_representable():
    R = _tiny_set()
    o = po.Oracle(R.m, R.n, 16, R.u, R.v, R.r, storage="fp16")
    o.train_epoch()
    P, Q = o.factors()
    for X in (P, Q):
        assert np.array_equal(X.astype(np.float16).astype(np.float32), X)


def test_create_rejects_bad_input():
    with pytest.raises(ValueError):
        po.Oracle(10, 10, 4, [10], [0], [1.0])
    with pytest.raises(ValueError):
        po.Oracle(10, 10, 4, [0], [0], [float("nan")])


# --------------------------------------------------------------------------- ADAGRAD (R23)

def test_adagrad_first_step_is_alpha_sign():
    """From zero accumulators each coordinate moves by exactly alpha against its gradient:
    dp / sqrt(dp^2) = sign(dp).  Dyadic values: exact.  p=(1,2), q=(3,4), r=10, lambda=.5:
    e = -1, dp = e q - l p = (-3.5, -5), dq = e p - l q = (-2.5, -4)."""
    p, q, gp, gq = po.update_adagrad([1, 2], [3, 4], [0, 0], [0, 0], 10.0, 0.125, 0.5, 0.5, eps=0.0)
    assert p.tolist() == [0.875, 1.875] and q.tolist() == [2.875, 3.875]
    assert gp.tolist() == [12.25, 25.0] and gq.tolist() == [6.25, 16.0]


def test_adagrad_reduces_to_plain_sgd_for_frozen_accumulators():
    """With accumulators at 2^40 an fp32 G + g^2 (g^2 < 2^16) stays 2^40 and sqrt(G) = 2^20, so
    the ADAGRAD step must equal Alg. 1's update with gamma = alpha * 2^-20 BIT-EXACTLY (scaling
    by a power of two commutes with rounding)."""
    rng = np.random.default_rng(8)
    for _ in range(50):
        k = int(rng.choice([1, 4, 16]))
        p = rng.normal(size=k).astype(np.float32)
        q = rng.normal(size=k).astype(np.float32)
        r, a = float(rng.normal() * 3), float(np.float32(rng.uniform(0.01, 1)))
        big = np.full(k, 2.0 ** 40, np.float32)
        p1, q1, gp, gq = po.update_adagrad(p, q, big, big, r, a, 0.05, 0.07, eps=0.0)
        p2, q2 = po.update(p, q, r, a * 2.0 ** -20, 0.05, 0.07)
        assert np.array_equal(p1, p2) and np.array_equal(q1, q2)
        assert np.array_equal(gp, big) and np.array_equal(gq, big)


def test_adagrad_step_direction_is_the_eq3_gradient():
    """(p' - p) sqrt(G') / alpha = -(1/2) grad_p of Eq. 3 (central differences, double)."""
    rng = np.random.default_rng(9)
    for _ in range(10):
        k = 7
        p = rng.normal(size=k).astype(np.float32)
        q = rng.normal(size=k).astype(np.float32)
        g0 = rng.uniform(0.5, 2.0, k).astype(np.float32)
        r, a, lp, lq = 1.3, 0.01, 0.2, 0.3
        p1, q1, gp, gq = po.update_adagrad(p, q, g0, g0, r, a, lp, lq, eps=0.0)
        pd, qd, h = p.astype(np.float64), q.astype(np.float64), 1e-6
        grad = np.array([(po.sample_loss(pd + h * e, qd, r, lp, lq) -
                          po.sample_loss(pd - h * e, qd, r, lp, lq)) / (2 * h) for e in np.eye(k)])
        step = (p1.astype(np.float64) - pd) * np.sqrt(gp.astype(np.float64)) / a
        np.testing.assert_allclose(step, -0.5 * grad, rtol=3e-3, atol=3e-3)


def test_adagrad_training_converges_on_tiny():
    R = _tiny_set()
    o = po.Oracle(R.m, R.n, 16, R.u, R.v, R.r, lambda_p=0.05, alpha=0.05, lr_rule="adagrad")
    r0 = o.rmse(R.ut, R.vt, R.rt)
    losses = [o.loss()]
    for _ in range(10):
        o.train_epoch()
        losses.append(o.loss())
    assert o.rmse(R.ut, R.vt, R.rt) < 0.5 * r0
    assert losses[-1] < 0.2 * losses[0]


# --------------------------------------------------------------------------- R24 grouped batches

def test_grouped_batches_order_hand_derived(golden_dir):
    """Reading R24: inside every batch of f consecutive samples the order is (relabelled
    column, storage position); the batch order itself is unchanged (A: S_HW)."""
    g = golden(golden_dir, "grouped_batches.json")
    cs = g["case"]
    u = np.array(cs["u"], np.int32)
    v = np.array(cs["v"], np.int32)
    r = np.ones(len(u), np.float32)
    o = po.Oracle(cs["m"], cs["n"], 16, u, v, r, seed=42, batch_f=cs["f"], group_cols=True)
    assert o.export("perm").tolist() == g["perm_S_SHUF_10"]
    assert o.export("rho_c").tolist() == g["rho_C"]
    assert o.export("chunkorder", 0).tolist() == g["chunk_order_t0"]
    assert o.export("order", 0).tolist() == g["order_grouped_t0"]
    plain = po.Oracle(cs["m"], cs["n"], 16, u, v, r, seed=42, batch_f=cs["f"])
    assert plain.export("order", 0).tolist() == g["order_plain_t0"]


def test_grouped_batches_permute_within_batches_only():
    """Property at any size: the grouped order is the plain order with each batch's samples
    permuted among themselves (same batches, same batch order, each sample once), and within a
    batch the relabelled columns are non-decreasing."""
    u, v, r, m, n = _tiny_uniform(m=97, n=13, N=4000)
    f = 64
    og = po.Oracle(m, n, 4, u, v, r, group_cols=True, seed=3, batch_f=f)
    op = po.Oracle(m, n, 4, u, v, r, seed=3, batch_f=f)
    a, b = og.export("order", 1), op.export("order", 1)
    assert sorted(a.tolist()) == list(range(4000))
    perm, rho_c = og.export("perm"), og.export("rho_c")
    pos = 0
    for q in og.export("chunkorder", 1):                  # one strata block: list = storage order
        batch = list(range(q * f, min(q * f + f, 4000)))
        assert b[pos:pos + len(batch)].tolist() == batch
        seg = a[pos:pos + len(batch)]
        assert sorted(seg.tolist()) == batch
        assert np.all(np.diff(rho_c[v[perm[seg]]]) >= 0)
        pos += len(batch)
    assert pos == 4000


# --------------------------------------------------------------------------- a x 1 row blocks (R27)

def test_row_block_grid_ids_hand_derived(golden_dir):
    """The paper's a x 1 grid (Hugewiki in 64 x 1 blocks; reading R27): a sample's block
    is its relabelled row segment alone.  On the App. A case (m = 10, n = 7, a = 2) every cell of
    row u lands in block row_of_u[u][0] of the hand derivation, whatever its column."""
    g, cs, o = _grid_case(golden_dir, schedule="hogwild", grid_cols=1)
    hb = np.empty(cs["N"], np.int64)
    hb[o.export("perm")] = o.export("blockid")
    want = [[ru[0]] * cs["n"] for ru in g["row_of_u"]]
    assert hb.reshape(cs["m"], cs["n"]).tolist() == want
    # the a x a grid's blocks of row segment r, merged, are the a x 1 block r
    _, _, oa = _grid_case(golden_dir, schedule="hogwild")
    ha = np.empty(cs["N"], np.int64)
    ha[oa.export("perm")] = oa.export("blockid")
    assert np.array_equal(ha // cs["a"], hb)


def test_row_block_epoch_order_hand_derived(golden_dir):
    """Epoch order of the a x 1 grid: the blocks one after another in the order pi_t =
    perm(S_STRATA(t), a) of App. A (golden pi_0_a8), each block's chunks in perm(S_HW(t, b))
    order.  With f larger than any block every block is one chunk, so epoch 0 must visit block
    pi_0[0]'s samples in storage order, then block pi_0[1]'s, ... (rho_R of the golden)."""
    ga = golden(golden_dir, "appendix_a.json")
    m, n, a = 10, 7, 8
    u = np.repeat(np.arange(m, dtype=np.int32), n)
    v = np.tile(np.arange(n, dtype=np.int32), m)
    o = po.Oracle(m, n, 16, u, v, np.ones(m * n, np.float32), seed=ga["seed"], grid_a=a,
                  grid_cols=1, batch_f=256)
    rho = ga["rho_R_10"]
    seg = [rho[uu] * a // m for uu in range(m)]           # floor(a rho / m), A: segments
    perm = o.export("perm")                                # caller index i = 7u + v per position
    want = []
    for b in ga["pi_0_a8"]:
        want += [p for p in range(m * n) if seg[perm[p] // n] == b]
    assert o.export("order", 0).tolist() == want
    assert o.export("strata", 0).tolist() == ga["pi_0_a8"]


def test_row_block_grid_with_one_block_is_the_plain_epoch():
    """a = 1: the a x 1 and a x a grids are the same single block (one Hogwild epoch)."""
    u, v, r, m, n = _tiny_uniform()
    o1 = po.Oracle(m, n, 8, u, v, r, grid_a=1, batch_f=32)
    o2 = po.Oracle(m, n, 8, u, v, r, grid_a=1, grid_cols=1, batch_f=32)
    for _ in range(2):
        o1.train_epoch()
        o2.train_epoch()
    assert np.array_equal(o1.factors()[0], o2.factors()[0])
    assert np.array_equal(o1.factors()[1], o2.factors()[1])
    assert o2.export("order", 3).tolist() == o1.export("order", 3).tolist()


def test_row_block_grid_every_sample_once_and_more_blocks_than_columns():
    """a x 1 needs a <= m only (a may exceed n); every sample is visited once per epoch."""
    u, v, r, m, n = _tiny_uniform()
    a = n + 3
    assert a <= m
    o = po.Oracle(m, n, 8, u, v, r, grid_a=a, grid_cols=1, batch_f=16)
    for t in range(2):
        assert sorted(o.export("order", t).tolist()) == list(range(len(u)))
    with pytest.raises(Exception):
        po.Oracle(m, n, 8, u, v, r, grid_a=a)                # a x a still needs a <= n
