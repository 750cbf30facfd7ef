"""CPU pin of the bound the GPU pruned search uses: SURVEY O11's chain
bound plus the 1F1B bubble term, written out here from the DAG argument and checked to
never exceed the oracle's exact T (like P6 for O11), for every k <= K.  It is a
lower-bound formula only, so if it overshot, the pruned search could drop the optimum;
this test (and the GPU key-equality tests) would catch that."""
import numpy as np
import pytest

import synth


def _bubble_bound(f, b, comm, n, p, m, K, cuts):
    """max over stages x of: fill_x + m*(wF_x + wB_x) + tail_x
    + max(0, R_x - (p-1-x)*wF_x), R_x = floor(sum_{i>x} F_i / K) - (p-1-x) [K > 1]
    + sum_{i>x} B_i; wF_x = F_x + C_{x-1}, wB_x = B_x + C_x (receiver-side comm)."""
    e = [0] + list(cuts) + [n]
    F = [int(f[e[x]:e[x + 1]].sum()) for x in range(p)]
    B = [int(b[e[x]:e[x + 1]].sum()) for x in range(p)]
    C = [int(comm[e[x + 1] - 1]) if x < p - 1 else 0 for x in range(p)]
    wF = [F[x] + (C[x - 1] if x > 0 else 0) for x in range(p)]
    wB = [B[x] + C[x] for x in range(p)]
    best = 0
    fill = tail = 0
    for x in range(p):
        v = fill + m * (wF[x] + wB[x]) + tail
        if x < p - 1:
            w = p - 1 - x
            q = sum(F[x + 1:]) // K
            R = (q if K == 1 else max(q - w, 0)) + sum(B[x + 1:])
            v += max(0, R - w * wF[x])
        best = max(best, v)
        fill += F[x] // K + (C[x - 1] // K if x > 0 else 0)
        tail += wB[x]
    return best


def test_bubble_bound_never_exceeds_T(oracle_mod):
    tight = stronger = 0
    for seed in range(400):
        kind = ["uniform", "b3f", "huge", "small", "equal"][seed % 5]
        n = 5 + seed % 14
        f, b, a = synth.random_tables(3000 + seed, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        p = 2 + seed % min(n - 1, 7)
        m = p + seed % 6          # the pruned kernel runs with m >= p
        K = 1 + seed % 4
        cuts = synth.random_cuts(seed + 7, n, p, 1)[0]
        lb = _bubble_bound(f, b, M.comm, n, p, m, K, cuts)
        for k in range(1, K + 1):
            assert M.T(p, m, cuts, k=k) >= lb, (seed, n, p, m, K, k)
        stronger += lb > M.lower_bound(p, m, K, cuts)
        tight += M.T(p, m, cuts, k=1) == lb
    assert stronger > 0 and tight > 0


def test_bubble_bound_balanced_and_configs(oracle_mod):
    """Near-balanced partitions (restart starts around Algorithm 1, where the bubble term
    matters most) on random tables and on the five configs' tables: never above T."""
    cases = []
    for seed in range(60):
        kind = ["uniform", "b3f", "equal"][seed % 3]
        n = 10 + seed % 20
        f, b, a = synth.random_tables(3500 + seed, n, kind)
        cases.append((f, b, a, synth.link_for(kind), 2 + seed % 7, None, 1 + seed % 4))
    for cfg in (1, 2, 3, 4, 5):
        wl = synth.config(cfg)
        f, b, a = wl.arrays()
        cases.append((f, b, a, wl.link_bytes_per_s, wl.p, wl.m, max(wl.k_hi, 1)))
    for f, b, a, bw, p, m, K in cases:
        n = len(f)
        p = min(p, n)
        m = m or p + 3
        M = oracle_mod.Model(f, b, a, bw)
        for r in range(6):
            cuts = [int(x) for x in M.restart_start(p, 0x5EED, 2, r)]
            lb = _bubble_bound(f, b, M.comm, n, p, m, K, cuts)
            for k in sorted({1, K}):
                assert M.T(p, m, cuts, k=k) >= lb, (n, p, m, K, k, cuts)


def _last_stage_bound(f, b, comm, n, p, m, K, cuts):
    """The last-stage skip's bound: stage p-1's chain bound
    fill + m*(wF + wB) + tail with every C_{p-2} term dropped (the comm into the last
    stage, in wF_{p-1} and in tail); the other comms depend on c_1..c_{p-2} only."""
    e = [0] + list(cuts) + [n]
    F = [int(f[e[x]:e[x + 1]].sum()) for x in range(p)]
    B = [int(b[e[x]:e[x + 1]].sum()) for x in range(p)]
    C = [int(comm[e[x + 1] - 1]) for x in range(p - 1)]
    fill = sum(F[x] // K for x in range(p - 1)) + sum(C[x - 1] // K for x in range(1, p - 1))
    tail = sum(B[:p - 1]) + sum(C[:p - 2])
    return fill + m * (F[p - 1] + B[p - 1]) + tail


def test_last_stage_bound_below_T_and_monotone(oracle_mod):
    """Never above the oracle's T for any k <= K (the skip drops only candidates with
    L >= S > T_opt), and non-increasing in c_{p-1} with c_1..c_{p-2} fixed (so the failing
    c_{p-1} form a prefix of their range, which the kernel steps past)."""
    for seed in range(300):
        kind = ["uniform", "b3f", "huge", "small", "equal"][seed % 5]
        n = 5 + seed % 14
        f, b, a = synth.random_tables(5000 + seed, n, kind)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        p = 2 + seed % min(n - 1, 7)
        m = p + seed % 6
        K = 1 + seed % 4
        cuts = [int(x) for x in synth.random_cuts(seed + 11, n, p, 1)[0]]
        for k in range(1, K + 1):
            assert M.T(p, m, cuts, k=k) >= _last_stage_bound(f, b, M.comm, n, p, m, K, cuts), seed
        lo = cuts[-2] + 1 if p > 2 else 1
        seq = [_last_stage_bound(f, b, M.comm, n, p, m, K, cuts[:-1] + [c]) for c in range(lo, n)]
        assert all(x >= y for x, y in zip(seq, seq[1:])), (seed, seq)
