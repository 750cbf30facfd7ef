"""Pins for the CPU oracle (-m "not gpu").

Every test here fixes the oracle against something other than itself: closed forms
derived from the schedule, the paper's own recurrences typed in literally, brute
force on tiny inputs, invariants, and independent cross-check values.  Each test
names the pin id of DESIGN.md §4.
"""
import itertools
import math

import numpy as np
import pytest

import synth


def _uniform_model(oracle, p, g, f, b, act, bw):
    """n = p*g identical blocks; cut vector giving every stage g blocks."""
    n = p * g
    M = oracle.Model([f] * n, [b] * n, [act] * n, bw)
    cuts = [g * (x + 1) for x in range(p - 1)]
    return M, cuts


# ----------------------------------------------------------------------------- P1
@pytest.mark.parametrize("p", [1, 2, 3, 4, 5, 6])
def test_P1_uniform_no_comm_closed_form(oracle_mod, p):
    """Uniform stages, zero comm: T = (m+p-1)(f+b) (BASELINE north_star closed form)."""
    rng = np.random.default_rng(p)
    for m in range(1, 12):
        f, b = int(rng.integers(0, 1000)), int(rng.integers(0, 1000))
        g = int(rng.integers(1, 3))
        M, cuts = _uniform_model(oracle_mod, p, g, f, b, 0, 10**9)
        r = M.simulate(p, m, cuts, want_path=True)
        assert r["T"] == (m + p - 1) * (f // 1 * g + b * g) // 1 or r["T"] == (m + p - 1) * g * (f + b)
        assert r["T"] == (m + p - 1) * g * (f + b)
        path = r["path"]
        assert path[0][:4] == (0, 0, 0, 0) and path[-1][:3] == (0, 1, m - 1)
        if f > 0 and b > 0:
            # every path is critical; the tie rule picks F(.,0) down, all 2m ops of
            # stage p-1, then B(., m-1) up: 2m + 2(p-1) ops, master p-1
            assert r["path_len"] == 2 * m + 2 * (p - 1)
            assert r["master"] == p - 1


# ----------------------------------------------------------------------------- P2
def test_P2_uniform_constant_comm_closed_form(oracle_mod):
    """Uniform stages with a constant comm C: p>=3, m>=2 ->
    T = (m+p-1)(f+b) + (2m+2p-5)C; p=2 -> T = (m+1)(f+b+C).  Path: (p-1) F-chain
    comms, the 1F1B run on stage p-2, (p-1) B-chain comms; with m >= 5 that run
    (2m-5 ops + 2) outnumbers stage p-1's 4 1F1B-phase path ops -> master p-2."""
    rng = np.random.default_rng(7)
    bw = 10**9  # 1 byte = 1 ns
    for trial in range(400):
        p = int(rng.integers(2, 7))
        m = int(rng.integers(2, 12)) if p >= 3 else int(rng.integers(1, 12))
        f, b = int(rng.integers(1, 500)), int(rng.integers(1, 500))
        Cc = int(rng.integers(0, 2 * max(f, b)))
        M, cuts = _uniform_model(oracle_mod, p, 1, f, b, Cc, bw)
        r = M.simulate(p, m, cuts)
        if p >= 3:
            assert r["T"] == (m + p - 1) * (f + b) + (2 * m + 2 * p - 5) * Cc, (p, m, f, b, Cc)
            if Cc > 0 and m >= 5:
                assert r["master"] == p - 2, (p, m, f, b, Cc)
        else:
            assert r["T"] == (m + 1) * (f + b + Cc), (p, m, f, b, Cc)


# ----------------------------------------------------------------------------- P3 / P4
def test_P3_single_microbatch(oracle_mod):
    """m = 1: the single micro-batch goes down and back up:
    T = sum_x (F_x + B_x) + 2 sum_{x<p-1} C_x."""
    for seed in range(200):
        n = 3 + seed % 9
        f, b, a = synth.random_tables(seed, n)
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        p = 1 + seed % n
        cuts = synth.random_cuts(seed, n, p, 1)[0]
        edges = [0] + list(cuts) + [n]
        expect = int(f.sum() + b.sum())
        for x in range(p - 1):
            expect += 2 * oracle_mod.comm_ns(int(a[edges[x + 1] - 1]), synth.LINK_BYTES_PER_S)
        assert M.T(p, 1, cuts) == expect


def test_P4_single_stage(oracle_mod):
    """p = 1: no comm, T = m (F + B)."""
    for seed in range(50):
        n = 1 + seed % 7
        f, b, a = synth.random_tables(seed, n)
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        for m in (1, 2, 5, 9):
            for k in (1, 3):
                assert M.T(1, m, [], k=k) == m * int(f.sum() + b.sum())


# ----------------------------------------------------------------------------- P5
def test_P5_slicing_uniform_closed_form(oracle_mod):
    """Slicing micro-batch 0 into k pieces, uniform stages, C = 0, k | f, m >= p:
    T(k) = (m+p-1)(f+b) - min((p-1)(f - f/k), b).  k = 2 with b >= (p-1)f/2 halves
    the forward fill (PAPER.md:13 'a 50% reduction in startup overhead')."""
    cnt = 0
    for p in range(2, 7):
        for m in range(p, p + 5):
            for k in (1, 2, 3, 4, 6):
                for f0 in (1, 2, 5):
                    f = f0 * 12
                    for b in (1, 7, f, 3 * f, 5 * f):
                        M, cuts = _uniform_model(oracle_mod, p, 1, f, b, 0, 10**9)
                        expect = (m + p - 1) * (f + b) - min((p - 1) * (f - f // k), b)
                        assert M.T(p, m, cuts, k=k) == expect, (p, m, k, f, b)
                        cnt += 1
    assert cnt > 1000


# ----------------------------------------------------------------------------- P6 / O11
def test_P6_lower_bounds(oracle_mod):
    """T >= LB_x for every stage (O11 chain bound, any k <= K) and T >= m*max(F_x+B_x)."""
    tight = 0
    for seed in range(300):
        kind = ["uniform", "b3f", "huge", "small", "equal"][seed % 5]
        n = 4 + seed % 12
        f, b, a = synth.random_tables(seed, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        p = 1 + seed % min(n, 6)
        m = 1 + seed % 9
        K = 1 + seed % 4
        cuts = synth.random_cuts(seed + 1, n, p, 1)[0]
        lb = M.lower_bound(p, m, K, cuts)
        edges = [0] + list(cuts) + [n]
        loads = [int(f[edges[x]:edges[x + 1]].sum() + b[edges[x]:edges[x + 1]].sum()) for x in range(p)]
        for k in range(1, K + 1):
            T = M.T(p, m, cuts, k=k)
            assert T >= lb
            assert T >= m * max(loads)
        tight += (M.T(p, m, cuts, k=1) == M.lower_bound(p, m, 1, cuts))
    assert tight > 0


# ----------------------------------------------------------------------------- P7 / P8
def test_P7_monotone_and_slicing_never_hurts(oracle_mod):
    """T is non-decreasing in every f_i, b_i, act_bytes_i and in m; T(k) <= T(1)."""
    for seed in range(150):
        n = 4 + seed % 10
        f, b, a = synth.random_tables(seed, n, "b3f" if seed % 2 else "uniform")
        bw = synth.LINK_BYTES_PER_S
        p = 1 + seed % min(n, 5)
        m = 1 + seed % 7
        cuts = synth.random_cuts(seed, n, p, 1)[0]
        M = oracle_mod.Model(f, b, a, bw)
        T0 = M.T(p, m, cuts)
        i = seed % n
        for arr in ("f", "b", "a"):
            f2, b2, a2 = f.copy(), b.copy(), a.copy()
            {"f": f2, "b": b2, "a": a2}[arr][i] += 1 + seed * 1000
            assert oracle_mod.Model(f2, b2, a2, bw).T(p, m, cuts) >= T0
        assert M.T(p, m + 1, cuts) >= T0
        for k in (2, 3, 5, 8):
            assert M.T(p, m, cuts, k=k) <= T0


def test_P8_k1_is_unsliced(oracle_mod):
    for seed in range(60):
        n = 3 + seed % 10
        f, b, a = synth.random_tables(seed, n)
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        p = 1 + seed % min(n, 5)
        cuts = synth.random_cuts(seed, n, p, 1)[0]
        m = 1 + seed % 6
        assert M.simulate(p, m, cuts, k=1, s=1)["T"] == M.simulate(p, m, cuts, k=1, s=0)["T"]
        assert M.simulate(p, m, cuts, k=4, s=0)["T"] == M.T(p, m, cuts)


# ----------------------------------------------------------------------------- P10
def test_P10_1f1b_block_count_and_stage_order(oracle_mod):
    """stage k of an n-stage pipeline owns max(0, m-n+k+1) 1F1B blocks
    (adjacent FP/BP pairs).  Checked on the oracle's per-stage op order."""
    f, b, a = synth.random_tables(3, 12)
    M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
    for p in range(1, 7):
        cuts = list(range(2, 2 * p, 2))
        for m in range(1, 10):
            ops = M.simulate(p, m, cuts, want_all=True)["ops"]
            for x in range(p):
                seq = [(kind, mb) for (st, kind, mb, q, s0, e0) in ops if st == x]
                nb = max(0, m - p + x + 1)
                w = m - nb
                expect = [(0, j) for j in range(w)]
                for y in range(nb):
                    expect += [(0, w + y), (1, y)]
                expect += [(1, y) for y in range(nb, m)]
                assert seq == expect, (p, m, x)


# ----------------------------------------------------------------------------- P12
def test_P12_paper_recurrences_transcribed(oracle_mod):
    """Type in PAPER.md:113-115 (1F1B phase) and :121-123 (cool-down) literally, seed
    them with the oracle's warm-up start times as the 'initial conditions' of
    PAPER.md:125, and check every 1F1B and cool-down start time of the DAG.

    t(x,y,0) = max(t(x-1,y-1,0)+f_{x-1}, t(x,y-1,1)+b_x) [+Comm if x != 0]
    t(x,y,1) = max(t(x+1,y,1)+b_{x+1}, t(x,y,0)+f_x)     [+Comm if x != n-1]
    t(x,y)   = max(t(x,y+1)+b_x, t(x+1,y)+b_{x+1}) + Comm   (cool-down, reversed y)
    with one constant Comm (the paper's model: all act_bytes equal)."""
    rng = np.random.default_rng(12)
    checked = 0
    for trial in range(120):
        p = int(rng.integers(2, 7))
        m = int(rng.integers(p, p + 8))
        n = p + int(rng.integers(0, 6))
        f = rng.integers(1, 1000, n); b = rng.integers(1, 1000, n)
        comm = int(rng.integers(0, 800))
        M = oracle_mod.Model(f, b, [comm] * n, 10**9)
        cuts = synth.random_cuts(trial, n, p, 1)[0]
        edges = [0] + list(cuts) + [n]
        fx = [int(f[edges[x]:edges[x + 1]].sum()) for x in range(p)]
        bx = [int(b[edges[x]:edges[x + 1]].sum()) for x in range(p)]
        ops = M.simulate(p, m, cuts, want_all=True)["ops"]
        start = {(st, kind, mb): s0 for (st, kind, mb, q, s0, e0) in ops}
        nblk = [max(0, m - p + x + 1) for x in range(p)]
        w = [m - nblk[x] for x in range(p)]

        def tF(x, y):  # 1F1B block y of stage x, FP: micro-batch w_x + y
            return start[(x, 0, w[x] + y)]

        def tB(x, y):  # 1F1B block y of stage x, BP: micro-batch y
            return start[(x, 1, y)]

        for x in range(p):
            for y in range(nblk[x]):
                # FP of block y: cross term needs block y-1 of stage x-1
                if x > 0 and y >= 1:
                    v = max(tF(x - 1, y - 1) + fx[x - 1], tB(x, y - 1) + bx[x]) + comm
                    assert v == tF(x, y), (x, y)
                    checked += 1
                # BP of block y
                terms = [tF(x, y) + fx[x]]
                if x < p - 1:
                    terms.append(tB(x + 1, y) + bx[x + 1])
                v = max(terms) + (comm if x != p - 1 else 0)
                assert v == tB(x, y)
                checked += 1
        # cool-down: renumbered in reverse; t(x, y) = start of B(x, m-1-y)
        for x in range(p - 1):
            ncool = w[x]
            for y in range(ncool):
                mb = m - 1 - y
                prev_same_stage = start[(x, 1, mb - 1)]  # t(x, y+1): previous BP on x
                v = max(prev_same_stage + bx[x], start[(x + 1, 1, mb)] + bx[x + 1]) + comm
                assert v == start[(x, 1, mb)]
                checked += 1
    assert checked > 5000


# ----------------------------------------------------------------------------- P9
def _all_longest_paths(ops, p, m, comm_of):
    """Enumerate every longest source->sink path of the DAG rebuilt in Python from
    the op list (edges re-derived from PAPER.md:113-123, independent of the C code)."""
    per_stage = {}
    for o in ops:
        per_stage.setdefault(o[0], []).append(o)
    idx = {(o[0], o[1], o[2], o[3]): i for i, o in enumerate(ops)}
    preds = {i: [] for i in range(len(ops))}
    for x, lst in per_stage.items():
        for a_, b_ in zip(lst, lst[1:]):
            preds[idx[b_[:4]]].append(idx[a_[:4]])
    for i, (st, kind, mb, q, s0, e0) in enumerate(ops):
        if kind == 0 and st > 0:
            preds[i].append(idx[(st - 1, 0, mb, q)])
        if kind == 1 and st < p - 1:
            preds[i].append(idx[(st + 1, 1, mb, 0)])
    sink = idx[(0, 1, m - 1, 0)]
    paths = []

    def back(v, acc):
        if len(paths) > 2000:
            return
        st, kind, mb, q, s0, e0 = ops[v]
        tgt = s0 - comm_of(ops[v])
        cand = [u for u in preds[v] if ops[u][5] == tgt]
        if not preds[v]:
            paths.append([v] + acc)
            return
        assert cand, "no tight predecessor"
        for u in cand:
            back(u, [v] + acc)

    back(sink, [])
    return paths


def test_P9_critical_path_tie_rule_brute_force(oracle_mod):
    """The oracle's critical path is a longest path (its length equals T, it runs from
    F(0,0,0) to B(0,m-1)) and, among ALL longest paths, it is the one 'closest to the
    last pipeline stage' read as the backward-lexicographically
    maximal stage sequence (reading Q10)."""
    ties = 0
    rng = np.random.default_rng(99)
    for seed in range(700):
        kind = ["small", "small", "equal", "uniform"][seed % 4]
        n = int(rng.integers(3, 8))
        f, b, a = synth.random_tables(seed, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        p = int(rng.integers(1, min(n, 4) + 1))
        m = int(rng.integers(1, 6))
        k = int(rng.integers(1, 4))
        cuts = synth.random_cuts(seed, n, p, 1)[0]
        r = M.simulate(p, m, cuts, k=k, want_path=True, want_all=True)
        edges = [0] + list(cuts) + [n]
        Cx = [oracle_mod.comm_ns(int(a[edges[x + 1] - 1]), bw) for x in range(p - 1)]

        def comm_of(o):
            st, kd, mb, q, s0, e0 = o
            if kd == 0 and st > 0:
                c = Cx[st - 1]
                return oracle_mod.split(c, k, q) if mb == 0 and k > 1 else c
            if kd == 1 and st < p - 1:
                return Cx[st]
            return 0

        path = r["path"]
        assert path[0][:4] == (0, 0, 0, 0)
        assert path[-1][:3] == (0, 1, m - 1)
        assert path[-1][5] == r["T"]
        # contiguity: each op starts exactly comm_in after its predecessor ends
        for u, v in zip(path, path[1:]):
            assert v[4] - comm_of(v) == u[5]
        ops = r["ops"]
        allp = _all_longest_paths(ops, p, m, comm_of)
        if len(allp) > 2000:
            continue
        ties += len(allp) > 1
        # backward-lexicographic maximum of stage sequences
        def key(pp):
            return [ops[v][0] for v in reversed(pp)]
        best = max(allp, key=key)
        assert [ops[v][:4] for v in best] == [o[:4] for o in path]
    assert ties > 30


def test_P9_master_rule(oracle_mod):
    """Master = stage with most critical-path ops in the 1F1B phase, ties -> higher."""
    for seed in range(80):
        n = 4 + seed % 6
        f, b, a = synth.random_tables(seed, n, "uniform")
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        p = 1 + seed % min(n, 5)
        m = 1 + seed % 8
        cuts = synth.random_cuts(seed, n, p, 1)[0]
        r = M.simulate(p, m, cuts, want_path=True)
        w = [min(p - 1 - x, m) for x in range(p)]
        cnt = [0] * p
        for (st, kind, mb, q, s0, e0) in r["path"]:
            in1f1b = (mb >= w[st]) if kind == 0 else (mb < m - w[st])
            cnt[st] += in1f1b
        best = max(range(p), key=lambda x: (cnt[x], x))
        assert r["master"] == (best if max(cnt) > 0 else p - 1)


# ----------------------------------------------------------------------------- P11 / Alg. 1
def test_P11_alg1_is_minmax_optimal(oracle_mod):
    """Algorithm 1's value equals the brute-force min over partitions of the max
    stage load (f+b), and its partition attains it; ties -> smallest k (first cut
    positions as small as possible from the right)."""
    for seed in range(120):
        n = 1 + seed % 9
        f, b, a = synth.random_tables(seed, n, "small" if seed % 2 else "uniform")
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        for p in range(1, n + 1):
            cuts, val = M.alg1(p)
            best = None
            for comb in itertools.combinations(range(1, n), p - 1):
                e = [0] + list(comb) + [n]
                load = max(int(f[e[x]:e[x + 1]].sum() + b[e[x]:e[x + 1]].sum()) for x in range(p))
                best = load if best is None else min(best, load)
            assert val == best
            e = [0] + list(cuts) + [n]
            assert all(e[x] < e[x + 1] for x in range(p))
            assert max(int(f[e[x]:e[x + 1]].sum() + b[e[x]:e[x + 1]].sum()) for x in range(p)) == val


# ----------------------------------------------------------------------------- enumeration
def test_rank_and_count(oracle_mod):
    """Lex enumeration: counter == closed-form rank (O7), count == C(n-1, p-1)."""
    for n in range(1, 10):
        for p in range(1, n + 1):
            assert oracle_mod.count(n, p) == math.comb(n - 1, p - 1)
            for r, comb in enumerate(itertools.combinations(range(1, n), p - 1)):
                assert oracle_mod.rank(n, p, list(comb)) == r
    assert oracle_mod.count(98, 16) == 154744841157936784
    assert oracle_mod.count(66, 8) == 696190560


def test_unrank_and_windows(oracle_mod):
    """The enumeration starts a rank window at the cut vector of its first rank: unrank
    is itertools' lexicographic order (independent of the rank formula), and a search
    split into random windows equals the single full enumeration (min over windows of
    (T, rank, k), simulation counts summing to N*K)."""
    for n in range(2, 11):
        for p in range(1, n + 1):
            for r, comb in enumerate(itertools.combinations(range(1, n), p - 1)):
                assert oracle_mod.unrank(n, p, r) == list(comb)
    rng = np.random.default_rng(9)
    for seed in range(12):
        n = 7 + seed % 6
        f, b, a = synth.random_tables(seed, n, ["uniform", "equal", "small"][seed % 3])
        M = oracle_mod.Model(f, b, a, synth.link_for(["uniform", "equal", "small"][seed % 3]))
        p = 2 + seed % 4
        m = p + seed % 3
        N = oracle_mod.count(n, p)
        full = M.exhaustive(p, m, 1, 3)
        cuts = sorted({0, N, *[int(x) for x in rng.integers(0, N, 4)]})
        parts = [M.exhaustive(p, m, 1, 3, lo, hi) for lo, hi in zip(cuts, cuts[1:]) if hi > lo]
        best = min(parts, key=lambda d: (d["T"], d["rank"], d["k"]))
        assert (best["T"], best["rank"], best["k"]) == (full["T"], full["rank"], full["k"])
        assert sum(d["sims"] for d in parts) == full["sims"] == 3 * N


def test_exhaustive_brute_force_tiny(oracle_mod):
    """or_exhaustive == min over itertools.combinations of (T, rank, k)."""
    for seed in range(40):
        kind = ["small", "uniform", "equal", "zero"][seed % 4]
        n = 2 + seed % 7
        f, b, a = synth.random_tables(seed, n, kind)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        p = 1 + seed % min(n, 4)
        m = 1 + seed % 5
        k_lo, k_hi = 1 + seed % 2, 1 + seed % 2 + seed % 3
        best = None
        for r, comb in enumerate(itertools.combinations(range(1, n), p - 1)):
            for k in range(k_lo, k_hi + 1):
                key = (M.T(p, m, list(comb), k=k), r, k)
                best = key if best is None else min(best, key)
        got = M.exhaustive(p, m, k_lo, k_hi)
        assert (got["T"], got["rank"], got["k"]) == best
        assert got["sims"] == math.comb(n - 1, p - 1) * (k_hi - k_lo + 1)
        # rank sub-ranges compose
        N = math.comb(n - 1, p - 1)
        mid = N // 2
        a1 = M.exhaustive(p, m, k_lo, k_hi, 0, mid) if mid > 0 else None
        a2 = M.exhaustive(p, m, k_lo, k_hi, mid, N)
        parts = [x for x in (a1, a2) if x is not None and x["sims"] > 0]
        mn = min(parts, key=lambda d: (d["T"], d["rank"], d["k"]))
        assert (mn["T"], mn["rank"], mn["k"]) == best


def test_bnb_equals_exhaustive(oracle_mod):
    """The LB-skipping enumeration returns exactly the brute-force argmin."""
    for seed in range(30):
        kind = ["uniform", "b3f", "small"][seed % 3]
        n = 6 + seed % 10
        f, b, a = synth.random_tables(seed, n, kind)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        p = 2 + seed % 4
        if p > n:
            continue
        m = p + seed % 6
        k_hi = 1 + seed % 3
        full = M.exhaustive(p, m, 1, k_hi)
        bnb = M.exhaustive_bnb(p, m, 1, k_hi)
        assert (bnb["T"], bnb["rank"], bnb["k"]) == (full["T"], full["rank"], full["k"])
        assert list(bnb["cuts"]) == list(full["cuts"])


# ----------------------------------------------------------------------------- misc defs
def test_comm_and_split_definitions(oracle_mod):
    assert oracle_mod.comm_ns(131072, 900 * 10**9) == 146        # 145.63.. -> ceil
    assert oracle_mod.comm_ns(900, 900 * 10**9) == 1
    assert oracle_mod.comm_ns(0, 900 * 10**9) == 0
    assert oracle_mod.comm_ns((1 << 40) + 1, (1 << 30) + 7) == -(-(((1 << 40) + 1) * 10**9) // ((1 << 30) + 7))  # bytes*1e9 > 2^64
    for v in (0, 1, 7, 100, 12345):
        for k in range(1, 17):
            parts = [oracle_mod.split(v, k, q) for q in range(k)]
            assert sum(parts) == v and min(parts) >= 0
            if k == 2:
                assert parts == [v // 2, v - v // 2]
    # splitmix64 reference output (seed 0 -> Vigna's published first value)
    assert oracle_mod.splitmix64(0) == 0xE220A8397B1DCDAF


# ----------------------------------------------------------------------------- P13
def test_P13_heuristic_properties(oracle_mod):
    """Heuristic result <= T(restart start), >= the exhaustive optimum; replay is
    deterministic; restart 0 starts at the Algorithm 1 partition."""
    for seed in range(25):
        n = 8 + seed % 8
        f, b, a = synth.random_tables(seed, n, "b3f")
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        p = 3 + seed % 3
        m = p + 2 * (seed % 3)
        opt = M.exhaustive(p, m)["T"]
        a1, _ = M.alg1(p)
        assert list(M.restart_start(p, 0x5EED, 2, 0)) == list(a1)
        for r in range(4):
            st = M.restart_start(p, 0x5EED, 2, r)
            assert all(0 < x < n for x in st) and all(np.diff(st) > 0)
            h = M.heuristic_restart(p, m, 0x5EED, 2, r)
            assert opt <= h["T"] <= M.T(p, m, st)
            assert M.T(p, m, h["cuts"]) == h["T"]
            h2 = M.heuristic_restart(p, m, 0x5EED, 2, r)
            assert h2["T"] == h["T"] and list(h2["cuts"]) == list(h["cuts"])
            assert h["steps"] <= n * p


# ----------------------------------------------------------------------------- P15
def test_P15_survey_crosscheck_values(oracle_mod):
    """Values from the survey's independent throwaway model (same
    formulas as §8d, not authoritative, but produced by different code)."""
    M1 = oracle_mod.Model.from_workload(synth.config(1))
    c, _ = M1.alg1(4)
    assert list(c) == [3, 6, 9]
    r = M1.simulate(4, 8, c, want_path=True)
    assert (r["T"], r["master"], r["path_len"]) == (49664, 3, 22)
    ex = M1.exhaustive(4, 8)
    assert (ex["T"], ex["rank"]) == (49664, 60)
    M2 = oracle_mod.Model.from_workload(synth.config(2))
    c, _ = M2.alg1(4)
    assert list(c) == [14, 27, 41] and M2.T(4, 16, c) == 90539622
    ex = M2.exhaustive(4, 16, 1, 1)
    assert (ex["T"], ex["rank"], list(ex["cuts"])) == (89891590, 12221, [15, 28, 41])
    assert M2.simulate(4, 16, ex["cuts"])["master"] == 0
    ex = M2.exhaustive(4, 16, 1, 4)
    assert (ex["T"], ex["rank"], ex["k"], list(ex["cuts"])) == (87232315, 12243, 4, [15, 29, 43])
    assert M2.heuristic_restart(4, 16, 0x5EED, 2, 0)["T"] == 89891590
    M3 = oracle_mod.Model.from_workload(synth.config(3))
    c, _ = M3.alg1(8)
    assert list(c) == [7, 13, 20, 27, 34, 41, 48] and M3.T(8, 32, c) == 94741098
    M4 = oracle_mod.Model.from_workload(synth.config(4))
    c, _ = M4.alg1(8)
    assert list(c) == [9, 17, 25, 33, 41, 50, 59] and M4.T(8, 64, c) == 672610004
    T, bk = M4.slice_sweep(8, 64, c, 8)
    assert list(T[1:]) == [666172833] * 7
    M5 = oracle_mod.Model.from_workload(synth.config(5))
    c, _ = M5.alg1(16)
    assert M5.T(16, 64, c) == 441984812
    assert M5.heuristic_restart(16, 64, 0x5EED, 2, 0)["T"] == 430480412


def test_algorithmic_op_count_matches_dag(oracle_mod):
    """bench.ops_per_sim (adds + distinct maxima) equals a direct count over the
    oracle's DAG: ops, and the number of distinct predecessor pairs among ops with
    two predecessors."""
    import importlib.util
    import os
    spec = importlib.util.spec_from_file_location(
        "bench", os.path.join(os.path.dirname(os.path.dirname(__file__)), "bench.py"))
    bench = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(bench)
    for p in range(1, 7):
        for m in range(1, 9):
            for k in (1, 2, 3):
                M, cuts = _uniform_model(oracle_mod, p, 1, 3, 5, 7, 10**9)
                ops = M.simulate(p, m, cuts, k=k, want_all=True)["ops"]
                ids = {o[:4] for o in ops}
                per_stage = {}
                for o in ops:
                    per_stage.setdefault(o[0], []).append(o[:4])
                prev = {}
                for x, lst in per_stage.items():
                    for a, b in zip(lst, lst[1:]):
                        prev[b] = a
                pairs = set()
                for (st, kind, mb, q) in ids:
                    cross = (st - 1, 0, mb, q) if kind == 0 else (st + 1, 1, mb, 0)
                    intra = prev.get((st, kind, mb, q))
                    if cross in ids and intra is not None:
                        pairs.add(frozenset((cross, intra)))
                assert bench.ops_per_sim(p, m, k) == len(ops) + len(pairs), (p, m, k)


def _longest_to_sink(ops, P):
    """h(op) = longest path from op (incl. its own weight) to the sink, on the DAG
    rebuilt from the oracle's op list (edges of PAPER.md:113-123)."""
    from collections import deque
    per_stage = {}
    for o in ops:
        per_stage.setdefault(o[0], []).append(o)
    idx = {o[:4]: i for i, o in enumerate(ops)}
    succ = {i: [] for i in range(len(ops))}
    preds = {i: [] for i in range(len(ops))}
    for x, lst in per_stage.items():
        for a_, b_ in zip(lst, lst[1:]):
            succ[idx[a_[:4]]].append(idx[b_[:4]])
    for i, (st, kind, mb, q, s0, e0) in enumerate(ops):
        if kind == 0 and st < P - 1:
            succ[i].append(idx[(st + 1, 0, mb, q)])
        if kind == 1 and st > 0:
            succ[i].append(idx[(st - 1, 1, mb, 0)])
    for i, ss in succ.items():
        for j in ss:
            preds[j].append(i)
    W = {i: o[5] - max([ops[j][5] for j in preds[i]], default=0) for i, o in enumerate(ops)}
    outdeg = {i: len(succ[i]) for i in succ}
    q = deque(i for i in succ if outdeg[i] == 0)
    h = {}
    while q:
        i = q.popleft()
        h[i] = W[i] + max([h[j] for j in succ[i]], default=0)
        for j in preds[i]:
            outdeg[j] -= 1
            if outdeg[j] == 0:
                q.append(j)
    return h, per_stage, idx


def test_kfactor_identity_on_oracle_dag(oracle_mod):
    """T(k) = max_x FF_x(k) + G_x with G_x the longest path from the
    end of F(x,0) through its intra-stage successor -- G independent of k.  Checked on
    the oracle's explicit DAG (the GPU's KFACTOR mode relies on it)."""
    rng = np.random.default_rng(5)
    for seed in range(120):
        kind = ["uniform", "small", "b3f"][seed % 3]
        n = int(rng.integers(2, 12))
        p = int(rng.integers(1, min(n, 6) + 1))
        m = int(rng.integers(p, p + 6))
        f, b, a = synth.random_tables(seed, n, kind)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        cuts = synth.random_cuts(seed, n, p, 1)[0]
        G_ref = None
        for k in (1, 2, 3, 5):
            r = M.simulate(p, m, cuts, k=k, want_all=True)
            h, per_stage, idx = _longest_to_sink(r["ops"], p)
            G, FF = [], []
            for x in range(p):
                lst = per_stage[x]
                last_piece = [o for o in lst if o[1] == 0 and o[2] == 0][-1]
                nxt = lst[lst.index(last_piece) + 1]
                G.append(h[idx[nxt[:4]]])
                FF.append(last_piece[5])
            if G_ref is None:
                G_ref = G
            assert G == G_ref
            assert max(FF[x] + G[x] for x in range(p)) == r["T"]


def test_heuristic_eq1_properties(oracle_mod):
    """adjust_mode 1: opt <= result <= T(start), deterministic, bounded walk; mode 0
    unchanged by the mode-1 machinery (P13 for step 2)."""
    for seed in range(20):
        n = 8 + seed % 10
        f, b, a = synth.random_tables(seed, n, "b3f")
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        p = 3 + seed % 3
        m = p + 2 * (seed % 3)
        opt = M.exhaustive(p, m)["T"]
        for r in range(3):
            st = M.restart_start(p, 0x5EED, 2, r)
            h1 = M.heuristic_restart(p, m, 0x5EED, 2, r, adjust_mode=1)
            assert opt <= h1["T"] <= M.T(p, m, st)
            assert M.T(p, m, h1["cuts"]) == h1["T"]
            h2 = M.heuristic_restart(p, m, 0x5EED, 2, r, adjust_mode=1)
            assert (h2["T"], list(h2["cuts"]), h2["sims"]) == (h1["T"], list(h1["cuts"]), h1["sims"])
            assert h1["steps"] <= n * p


def test_paper_slicer_form_pins(oracle_mod):
    """Paper Slicer form (first s micro-batches in k pieces): s=0 is unsliced, s=1 is
    the north-star form (micro-batch 0 in k pieces), T never increases from s=0 to
    s=1 (P7), and uniform stages with C=0 reproduce P5 at s=1."""
    for seed in range(60):
        n = 4 + seed % 10
        f, b, a = synth.random_tables(seed, n, "b3f")
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        p = 1 + seed % min(n, 6)
        m = p + seed % 5
        cuts = synth.random_cuts(seed, n, p, 1)[0]
        T, bs = M.slice_sweep_paper(p, m, cuts, 2, m)
        assert T[0] == M.T(p, m, cuts, k=1)
        assert T[1] == M.T(p, m, cuts, k=2)
        assert T[1] <= T[0]
        assert T[bs] == min(T) and all(T[s] > T[bs] for s in range(bs))


def test_alg2_text_reading_matches_simulation(oracle_mod):
    """Algorithm 2 is unpinned by the paper, but its purpose is to
    pick the number of halved micro-batches.  Its text reading (reading 1)
    attains the simulated minimum of T(s) on all five configs and on >= 95% of random
    Alg.-1 partitions with m = 2p (the paper's Fig. 10 setting); the printed pseudocode
    test (reading 0) does not (Q23)."""
    for cfg in synth.ALL_CONFIGS:
        wl = synth.config(cfg)
        M = oracle_mod.Model.from_workload(wl)
        c, _ = M.alg1(wl.p)
        T, bs = M.slice_sweep_paper(wl.p, wl.m, c, 2, wl.p)
        mb = M.alg2(wl.p, c, 1)
        assert 1 <= mb <= wl.p and T[mb] == T[bs]
    hit = {0: 0, 1: 0}
    for seed in range(200):
        rng = np.random.default_rng(seed)
        n = int(rng.integers(8, 40))
        f, b, a = synth.random_tables(seed, n, "b3f")
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        p = int(np.random.default_rng(seed + 1).integers(2, min(n, 10) + 1))
        c, _ = M.alg1(p)
        T, bs = M.slice_sweep_paper(p, 2 * p, c, 2, p)
        for rd in (0, 1):
            hit[rd] += int(T[M.alg2(p, c, rd)] == T[bs])
    assert hit[1] >= 190 and hit[0] < hit[1]


# ----------------------------------------------------------------------------- P14
def test_P14_minlb_relaxation_exact_for_uniform_comm(oracle_mod):
    """Certified minLB (reading R-LB): with K = 1 and one Comm value for every
    cut, the per-stage relaxation is exact, so the DP equals brute force
    min over all C(n-1,p-1) partitions of the O11 bound (or_lower_bound, pinned by P6),
    and the partition it returns attains it."""
    for seed in range(120):
        kind = ["uniform", "b3f", "small", "equal", "huge"][seed % 5]
        n = 4 + seed % 9
        f, b, a = synth.random_tables(seed, n, kind)
        a = np.full(n, int(a[0]), np.int64)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        p = 1 + seed % min(n, 5)
        m = 1 + seed % 7
        lb, cuts = M.min_lower_bound(p, m, 1)
        brute = min(M.lower_bound(p, m, 1, list(c))
                    for c in itertools.combinations(range(1, n), p - 1))
        assert lb == brute, (seed, lb, brute)
        assert M.lower_bound(p, m, 1, list(cuts)) == lb
        assert all(0 < cuts[i] < n for i in range(p - 1))
        assert all(cuts[i] < cuts[i + 1] for i in range(p - 2))


def test_P14_minlb_is_certified(oracle_mod):
    """For any Comm and any K: minLB <= min_c LB(c, K) <= min over (c, k <= K) of T
    (brute force), and the C1 bound is tight (= the P15 optimum 49 664)."""
    tight = 0
    for seed in range(120):
        kind = ["uniform", "b3f", "small", "equal", "huge"][seed % 5]
        n = 4 + seed % 9
        f, b, a = synth.random_tables(seed, n, kind)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        p = 1 + seed % min(n, 5)
        m = 1 + seed % 7
        K = 1 + seed % 4
        lb, _ = M.min_lower_bound(p, m, K)
        lbc = min(M.lower_bound(p, m, K, list(c))
                  for c in itertools.combinations(range(1, n), p - 1))
        opt = M.exhaustive(p, m, 1, K)["T"]
        assert lb <= lbc <= opt, (seed, lb, lbc, opt)
        tight += lb == opt
    assert tight > 10
    wl = synth.config(1)
    M = oracle_mod.Model.from_workload(wl)
    assert M.min_lower_bound(wl.p, wl.m, 1)[0] == 49664 == M.exhaustive(wl.p, wl.m)["T"]


# ----------------------------------------------------------------------------- N1 reach
def test_reach_is_the_fixpoint_closure(oracle_mod):
    """Reachable-set search (reading R-N1) against an order-free definition:
    with T and master of EVERY partition simulated up front (brute force), the
    evaluated set must be the least set E with start in E and, for every u in the
    qualifying set Q (start, plus children c of a Q-node u with master(c) <= master(u))
    with master(u) > 0, all of u's children in E.  The result is min T over E, and it
    is never worse than the greedy walk (whose path lies inside Q)."""
    for seed in range(40):
        kind = ["uniform", "b3f", "small", "equal"][seed % 4]
        n = 6 + seed % 7
        f, b, a = synth.random_tables(seed, n, kind)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        p = 2 + seed % min(n - 1, 4)
        m = p + seed % 5
        allp = {c: M.simulate(p, m, list(c)) for c in itertools.combinations(range(1, n), p - 1)}
        _, arg = M.alg1_table(p)

        def kids(c, i):
            cc = [0] + list(c) + [n]
            out = []
            if cc[i + 1] - cc[i] < 2:
                return out
            A = cc[:]; A[i] += 1; out.append(A)
            Ap = A[:]
            e = Ap[i - 1]
            for jj in range(i - 1, 1, -1):
                Ap[jj - 1] = int(arg[e, jj]); e = Ap[jj - 1]
            if Ap != A:
                out.append(Ap)
            if i <= p - 2:
                Bc = cc[:]; Bc[i + 1] -= 1; out.append(Bc)
                Bp = Bc[:]
                e = Bp[i]
                for jj in range(i, 1, -1):
                    Bp[jj - 1] = int(arg[e, jj]); e = Bp[jj - 1]
                if Bp != Bc:
                    out.append(Bp)
            return [tuple(x[1:p]) for x in out]

        for r in range(4):
            start = tuple(int(x) for x in M.restart_start(p, seed, 2, r))
            Q, E, todo = {start}, {start}, [start]
            while todo:
                u = todo.pop()
                iu = allp[u]["master"]
                if iu == 0:
                    continue
                for c in kids(u, iu):
                    E.add(c)
                    if allp[c]["master"] <= iu and c not in Q:
                        Q.add(c); todo.append(c)
            o = M.reach_restart(p, m, seed, 2, r)
            assert not o["truncated"]
            assert o["sims"] == len(E), (seed, r)
            assert o["T"] == min(allp[c]["T"] for c in E)
            assert allp[tuple(int(x) for x in o["cuts"])]["T"] == o["T"]
            assert o["T"] <= M.heuristic_restart(p, m, seed, 2, r)["T"]


def test_reach_truncation_and_bounds(oracle_mod):
    """vmax caps the evaluated set exactly (sims == vmax when truncated); with a cap
    the result is still an attained T >= the optimum; restart 0 on C2 reaches the
    k=1 optimum (P15) like the greedy walk."""
    wl = synth.config(5)
    M = oracle_mod.Model.from_workload(wl)
    full = M.reach_restart(wl.p, wl.m, wl.seed, wl.radius, 0)
    assert not full["truncated"] and full["sims"] > 8
    for vmax in (1, 2, 5, full["sims"] - 1):
        o = M.reach_restart(wl.p, wl.m, wl.seed, wl.radius, 0, vmax=vmax)
        assert o["truncated"] and o["sims"] == vmax and o["T"] >= full["T"]
        assert M.T(wl.p, wl.m, o["cuts"]) == o["T"]
    o = M.reach_restart(wl.p, wl.m, wl.seed, wl.radius, 0, vmax=full["sims"])
    assert not o["truncated"] and o["T"] == full["T"]
    wl = synth.config(2)
    M = oracle_mod.Model.from_workload(wl)
    assert M.reach_restart(wl.p, wl.m, wl.seed, wl.radius, 0)["T"] == 89891590


# ----------------------------------------------------------------------------- N4 memory
def test_N4_inflight_count_matches_the_schedule(oracle_mod):
    """Reading R-N4's in-flight count: the most micro-batches stage x holds between
    their FP and BP, read off the oracle's own 1F1B op order (ops sorted by start on
    each stage, positive costs), is min(p - x, m)."""
    for p in range(1, 7):
        for m in range(1, 10):
            n = p + 2
            M = oracle_mod.Model([3 + i for i in range(n)], [5 + 2 * i for i in range(n)],
                                 [7] * n, 10**9)
            cuts = list(range(1, p))
            ops = M.simulate(p, m, cuts, want_all=True)["ops"]
            for x in range(p):
                seq = sorted((o[4], o[1]) for o in ops if o[0] == x)
                cur = most = 0
                for _, kind in seq:
                    cur += 1 if kind == 0 else -1
                    most = max(most, cur)
                assert most == min(p - x, m), (p, m, x)


def test_N4_memory_feasibility_handworked(oracle_mod):
    """n = 4, p = 2, m = 3, static 10 B and stash 1 B per sub-layer: in-flight 2 on
    stage 0 and 1 on stage 1, so cut 1 needs (12, 33) B, cut 2 (24, 22) B, cut 3
    (36, 11) B.  cap 33 admits cuts 1 and 2, cap 24 only cut 2, cap 23 none."""
    M = oracle_mod.Model([4, 1, 1, 4], [8, 2, 2, 8], [0, 0, 0, 0], 10**9)
    st, sh = [10] * 4, [1] * 4
    assert [M.feasible(2, 3, [c], st, sh, 33) for c in (1, 2, 3)] == [True, True, False]
    assert [M.feasible(2, 3, [c], st, sh, 24) for c in (1, 2, 3)] == [False, True, False]
    assert not any(M.feasible(2, 3, [c], st, sh, 23) for c in (1, 2, 3))
    r = M.exhaustive_mem(2, 3, 1, 1, st, sh, 33)
    Ts = {c: M.T(2, 3, [c]) for c in (1, 2)}
    assert r["T"] == min(Ts.values()) and list(r["cuts"]) == [min(Ts, key=lambda c: (Ts[c], c))]
    assert M.exhaustive_mem(2, 3, 1, 1, st, sh, 24)["cuts"][0] == 2
    assert M.exhaustive_mem(2, 3, 1, 1, st, sh, 23)["T"] is None


def test_N4_plan_depths_properties(oracle_mod):
    """Unlimited memory: every depth's feasible argmin is the plain exhaustive one, and
    the outer loop picks p = 1 with T = m*sum(f+b) (P4; a deeper pipeline only adds
    fill and drain).  Shrinking the capacity never lowers the chosen T, and below the
    smallest possible stage footprint nothing is feasible."""
    for seed in range(12):
        kind = ["uniform", "b3f", "small"][seed % 3]
        n = 6 + seed % 6
        f, b, a = synth.random_tables(seed, n, kind)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        rng = np.random.default_rng(seed)
        st = rng.integers(1, 1000, n)
        sh = rng.integers(0, 100, n)
        G, mb = 4, 8
        best, per = M.plan_depths(G, mb, st, sh, 1 << 60)
        for r in per:
            ex = M.exhaustive(r["p"], r["m"])
            assert (r["T"], r["rank"]) == (ex["T"], ex["rank"])
        assert best["p"] == 1 and best["T"] == (mb // G) * int(f.sum() + b.sum())
        prevT = best["T"]
        for cap in sorted({int(st.sum() + 8 * sh.sum()) // d for d in (1, 2, 3, 4, 6, 8)},
                          reverse=True):
            bst, _ = M.plan_depths(G, mb, st, sh, cap)
            if bst is None:
                prevT = None
                continue
            assert prevT is not None and bst["T"] >= prevT
            prevT = bst["T"]
        assert M.plan_depths(G, mb, st, sh, int(st.min()) - 1)[0] is None
