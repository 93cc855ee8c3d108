"""Critical path of the deterministic wavefront schedule (section 5.2 with (w,i) tickets, R10).

Visit (w, i) runs sub-block (i, seq_i[w]).  It can start only when worker i finished wave w-1
AND the previous visit of the same column (lexicographic (w', i') < (w, i)) has released it:
    finish(w,i) = max(finish(w-1,i), finish(prev visit of column)) + t_handoff + n(i,j) * t_upd
The epoch time of ANY implementation of this schedule is >= max finish (plus the
bandwidth floor).  Sub-block sizes come from Netflix-shaped synthetic data (SURVEY 8(d) skew).

    python tools/wf_critical_path.py [--s 1024] [--c 2048] [--t-upd 100e-9] [--t-hand 1e-6]
        [--cyclic] [--fraction 0.25]
"""
import argparse
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def subblock_counts(s, c, fraction, seed=1):
    import torch
    from paper_conf_hpdc_xietfl17_b200 import synth
    R = synth.shaped("netflix", fraction=fraction, device="cpu", with_test=False)
    rng = np.random.default_rng(seed)
    rho_r = rng.permutation(R.m)
    rho_c = rng.permutation(R.n)
    u = R.u.numpy().astype(np.int64)
    v = R.v.numpy().astype(np.int64)
    i = rho_r[u] * s // R.m
    j = rho_c[v] * c // R.n
    cnt = np.bincount(i * c + j, minlength=s * c).reshape(s, c)
    return cnt, R


def critical_path(cnt, seq, t_upd, t_hand):
    s, c = cnt.shape
    fin_worker = np.zeros(s)
    fin_col = np.zeros(c)
    for w in range(c):
        cols = seq[:, w]
        # workers in increasing i; conflicts inside a wave are serialised in i order
        for i in range(s):
            col = cols[i]
            start = max(fin_worker[i], fin_col[col])
            f = start + t_hand + cnt[i, col] * t_upd
            fin_worker[i] = f
            fin_col[col] = f
    return fin_worker.max()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--s", type=int, default=1024)
    ap.add_argument("--c", type=int, default=0)
    ap.add_argument("--t-upd", type=float, default=100e-9)
    ap.add_argument("--t-hand", type=float, default=1e-6)
    ap.add_argument("--cyclic", action="store_true")
    ap.add_argument("--fraction", type=float, default=1.0)
    a = ap.parse_args()
    c = a.c or 2 * a.s
    t0 = time.time()
    cnt, R = subblock_counts(a.s, c, a.fraction)
    scale = 1.0 / a.fraction              # counts scale with N (m, n scaled too: keep per-block)
    rng = np.random.default_rng(7)
    if a.cyclic:
        tau = rng.permutation(c)[:a.s]
        sigma = rng.permutation(c)
        seq = sigma[(tau[:, None] + np.arange(c)[None, :]) % c]
    else:
        seq = np.stack([rng.permutation(c) for _ in range(a.s)])
    cp = critical_path(cnt * scale, seq, a.t_upd, a.t_hand)
    col_tot = (cnt * scale).sum(0)
    print(f"s={a.s} c={c} cyclic={a.cyclic} t_upd={a.t_upd*1e9:.0f}ns t_hand={a.t_hand*1e6:.2f}us: "
          f"critical path {cp*1e3:.1f} ms; heaviest column block {col_tot.max():.0f} updates "
          f"-> chain floor {col_tot.max()*a.t_upd*1e3 + a.s*a.t_hand*1e3:.1f} ms; "
          f"mean sub-block {cnt.mean()*scale:.1f}; ({time.time()-t0:.0f}s)")


if __name__ == "__main__":
    main()
