"""GPU <-> oracle parity (-m gpu).  Bit-exact on every integer output.

Every GPU call goes through the C ABI (libap.so via the thin binding); every
expected value comes from oracle/ on the same seeded synth inputs.
"""
import math
import os

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ap():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_cluster_liulldgl22_b200 as ap
    return ap


def _plan(ap, f, b, a, bw):
    return ap.ap_plan_create(f, b, a, bw, device=0)


def _eval(ap, plan, p, m, cuts, ks, master=True):
    import torch
    cnt = len(cuts)
    c = torch.tensor(np.asarray(cuts, np.int32).reshape(cnt, max(p - 1, 0)), device="cuda")
    if p == 1:
        c = torch.zeros((cnt, 0), dtype=torch.int32, device="cuda")
    k = torch.tensor(np.asarray(ks, np.int32), device="cuda")
    T = torch.empty(cnt, dtype=torch.int64, device="cuda")
    M = torch.empty(cnt, dtype=torch.int32, device="cuda") if master else None
    ap.ap_eval_batch(plan, p, m, c, k, T, M)
    torch.cuda.synchronize()
    return T.cpu().numpy(), (M.cpu().numpy() if master else None)


# --------------------------------------------------------------------------- K2
@pytest.mark.parametrize("kind", ["uniform", "b3f", "small", "equal", "huge", "zero"])
def test_eval_batch_random_vs_oracle(ap, oracle_mod, kind):
    """Random (n, p, m, k, cuts) incl. m < p-1, ties, zero costs: T and master."""
    rng = np.random.default_rng(hash(kind) % 1000)
    for trial in range(12):
        n = int(rng.integers(2, 40))
        f, b, a = synth.random_tables(trial * 7 + len(kind), n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        for p in sorted({1, 2, int(rng.integers(1, min(n, 32) + 1)), min(n, 16)}):
            m = int(rng.choice([1, 2, 3, p - 1 if p > 1 else 1, p, p + 1, 2 * p + 3, 40]))
            cnt = 24
            cuts = synth.random_cuts(trial + 100 * p, n, p, cnt)
            ks = rng.integers(1, 17, cnt)
            T, Ms = _eval(ap, plan, p, m, cuts, ks)
            for i in range(cnt):
                r = M.simulate(p, m, cuts[i], k=int(ks[i]))
                assert T[i] == r["T"], (kind, n, p, m, int(ks[i]), list(cuts[i]))
                assert Ms[i] == r["master"], (kind, n, p, m, int(ks[i]), list(cuts[i]))


def test_eval_batch_invalid_rows(ap):
    import torch
    f, b, a = synth.random_tables(1, 10)
    plan = _plan(ap, f, b, a, synth.LINK_BYTES_PER_S)
    cuts = torch.tensor([[3, 5, 7], [5, 3, 7], [0, 3, 7], [3, 5, 10]], dtype=torch.int32, device="cuda")
    k = torch.tensor([1, 1, 1, 1], dtype=torch.int32, device="cuda")
    T = torch.empty(4, dtype=torch.int64, device="cuda")
    ap.ap_eval_batch(plan, 4, 8, cuts, k, T)
    assert T.cpu().tolist()[1:] == [-1, -1, -1] and T.cpu().tolist()[0] > 0


@pytest.mark.parametrize("p,m,with_master", [(4, 8, False), (4, 8, True), (3, 8, False),
                                             (4, 2, True)])
def test_eval_batch_ex_counts_invalid_rows(ap, oracle_mod, p, m, with_master):
    """ap_eval_batch_ex: the invalid-row count equals the rows written as -1, on the fast
    kernel (p = 4, m >= p), the generic one (p = 3; m < p) and with the master; valid
    rows still equal the oracle; a second call re-zeroes the count."""
    import torch
    f, b, a = synth.random_tables(7, 12)
    plan = _plan(ap, f, b, a, synth.LINK_BYTES_PER_S)
    M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
    rng = np.random.default_rng(11)
    rows, ks, bad = [], [], []
    for i in range(300):
        c = sorted(rng.choice(np.arange(1, 12), p - 1, replace=False).tolist())
        kk = int(rng.integers(1, 5))
        kind = i % 5
        if kind == 1:
            c[0] = 0                      # cut outside [1, n-1]
        elif kind == 2 and p - 1 >= 2:
            c[0], c[1] = c[1], c[0]       # not increasing
        elif kind == 3:
            kk = 17                       # k > AP_MAX_K
        rows.append(c)
        ks.append(kk)
        bad.append(kind in (1, 3) or (kind == 2 and p - 1 >= 2))
    cuts = torch.tensor(rows, dtype=torch.int32, device="cuda")
    k = torch.tensor(ks, dtype=torch.int32, device="cuda")
    T = torch.empty(len(rows), dtype=torch.int64, device="cuda")
    Ms = torch.empty(len(rows), dtype=torch.int32, device="cuda") if with_master else None
    nbad = torch.full((1,), 12345, dtype=torch.int64, device="cuda")
    for _ in range(2):
        ap.ap_eval_batch(plan, p, m, cuts, k, T, Ms, n_invalid=nbad)
        torch.cuda.synchronize()
        assert int(nbad.item()) == sum(bad)
    Th = T.cpu().tolist()
    Mh = Ms.cpu().tolist() if with_master else None
    for i, c in enumerate(rows):
        if bad[i]:
            assert Th[i] == -1 and (Mh is None or Mh[i] == -1)
        else:
            r = M.simulate(p, m, c, k=ks[i])
            assert Th[i] == r["T"]
            if Mh is not None:
                assert Mh[i] == r["master"]


def test_table2_partitions(ap, oracle_mod):
    """PAPER.md Table II partitions (GPT-2 345M, p=4) as named eval inputs."""
    import json
    doc = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table2_gpt2_345m.json")))
    wl = synth.config(2)
    f, b, a = wl.arrays()
    M = oracle_mod.Model(f, b, a, wl.link_bytes_per_s)
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    cuts = [prt["cuts"] for prt in doc["partitions"]]
    for m in (8, 16):
        T, Ms = _eval(ap, plan, 4, m, cuts, [1] * len(cuts))
        for i, c in enumerate(cuts):
            r = M.simulate(4, m, c)
            assert (T[i], Ms[i]) == (r["T"], r["master"])


# --------------------------------------------------------------------------- cpath
def test_critical_path_vs_oracle(ap, oracle_mod):
    rng = np.random.default_rng(5)
    for trial in range(40):
        kind = ["small", "uniform", "b3f"][trial % 3]
        n = int(rng.integers(2, 20))
        f, b, a = synth.random_tables(trial, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        p = int(rng.integers(1, min(n, 16) + 1))
        m = int(rng.integers(1, 12))
        k = int(rng.integers(1, 6))
        cuts = synth.random_cuts(trial, n, p, 1)[0]
        g = ap.ap_critical_path(plan, p, m, k, cuts)
        o = M.simulate(p, m, cuts, k=k, want_path=True)
        assert g["T"] == o["T"] and g["master"] == o["master"]
        assert g["path"] == o["path"], (n, p, m, k)


def test_critical_path_capacity(ap):
    f, b, a = synth.random_tables(3, 12)
    plan = _plan(ap, f, b, a, synth.LINK_BYTES_PER_S)
    with pytest.raises(ap.APError) as ei:
        ap.ap_critical_path(plan, 4, 8, 1, [3, 6, 9], cap=2)
    assert ei.value.status == 5


# --------------------------------------------------------------------------- Alg. 1
def test_alg1_vs_oracle(ap, oracle_mod):
    for seed in range(30):
        kind = ["uniform", "small", "equal"][seed % 3]
        n = 1 + (seed * 7) % 120
        f, b, a = synth.random_tables(seed, n, kind)
        M = oracle_mod.Model(f, b, a, synth.link_for(kind))
        plan = _plan(ap, f, b, a, synth.link_for(kind))
        for p in sorted({1, min(n, 2), min(n, 7), min(n, 16), min(n, 32)}):
            gc, gv = ap.ap_alg1(plan, p)
            oc, ov = M.alg1(p)
            assert list(gc) == list(oc) and gv == ov, (n, p)
    for i in synth.ALL_CONFIGS:
        wl = synth.config(i)
        f, b, a = wl.arrays()
        plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
        oc, ov = oracle_mod.Model.from_workload(wl).alg1(wl.p)
        gc, gv = ap.ap_alg1(plan, wl.p)
        assert list(gc) == list(oc) and gv == ov


# --------------------------------------------------------------------------- K1
def _search(ap, plan, p, m, k_lo, k_hi, lo=None, hi=None):
    import torch
    N = ap.ap_count(plan.n, p)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_search_exhaustive(plan, p, m, k_lo, k_hi, 0 if lo is None else lo, N if hi is None else hi, key)
    torch.cuda.synchronize()
    return int(key.item())


@pytest.mark.parametrize("mode", ["", "int64", "generic"])
def test_exhaustive_small_random_vs_oracle(ap, oracle_mod, mode, monkeypatch):
    if mode:
        monkeypatch.setenv("AP_SWEEP", mode)
    rng = np.random.default_rng(11)
    for trial in range(14):
        kind = ["uniform", "b3f", "small", "equal"][trial % 4]
        n = int(rng.integers(3, 16))
        f, b, a = synth.random_tables(trial, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        p = int(rng.integers(1, min(n, 6) + 1))
        m = int(rng.choice([1, 2, p, p + 3, 12]))
        k_lo = int(rng.integers(1, 3)); k_hi = k_lo + int(rng.integers(0, 4))
        key = _search(ap, plan, p, m, k_lo, k_hi)
        res = ap.ap_decode(plan, 0, p, m, k_lo, k_hi, key=key)
        o = M.exhaustive(p, m, k_lo, k_hi)
        assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"]), (n, p, m, k_lo, k_hi, mode)
        assert res["cuts"] == [int(x) for x in o["cuts"]]
        assert res["master"] == M.simulate(p, m, o["cuts"], k=o["k"])["master"]


@pytest.mark.parametrize("cfg", [1, 2])
def test_exhaustive_configs_full_vs_oracle(ap, oracle_mod, cfg):
    """C1 and C2 exactly: full oracle brute force vs the GPU sweep + decode."""
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    M = oracle_mod.Model.from_workload(wl)
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    key = _search(ap, plan, wl.p, wl.m, wl.k_lo, wl.k_hi)
    info = ap.ap_last_launch()
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=key)
    o = M.exhaustive_parallel(wl.p, wl.m, wl.k_lo, wl.k_hi)
    assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])
    assert info["fast_u32"] == 1 and info["exact_p"] == 1
    # k = 1 subproblem of C2 as well
    if cfg == 2:
        key = _search(ap, plan, 4, 16, 1, 1)
        res = ap.ap_decode(plan, 0, 4, 16, 1, 1, key=key)
        assert (res["time_ns"], res["rank"]) == (89891590, 12221)


@pytest.mark.parametrize("cfg", [3, 4])
def test_exhaustive_big_configs_vs_oracle_bnb(ap, oracle_mod, cfg):
    """C3 / C4 at full size, in the bench's launch configuration: the GPU argmin
    equals the oracle's exact argmin (its LB-skipping enumeration, same order)."""
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    M = oracle_mod.Model.from_workload(wl)
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    key = _search(ap, plan, wl.p, wl.m, wl.k_lo, wl.k_hi)
    info = ap.ap_last_launch()
    assert info["fast_u32"] == 1
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=key)
    o = M.exhaustive_bnb(wl.p, wl.m, wl.k_lo, wl.k_hi)
    assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])
    assert res["cuts"] == [int(x) for x in o["cuts"]]


def test_exhaustive_sampled_ranks_big(ap, oracle_mod):
    """C4 sampled: the GPU's argmin over many tiny rank windows (bench kernel,
    u32 path) equals the oracle's brute force over the same windows."""
    wl = synth.config(4)
    f, b, a = wl.arrays()
    M = oracle_mod.Model.from_workload(wl)
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    rng = np.random.default_rng(4)
    for lo in rng.integers(0, N - 40, 12):
        lo = int(lo)
        key = _search(ap, plan, wl.p, wl.m, 1, 8, lo, lo + 40)
        o = M.exhaustive(wl.p, wl.m, 1, 8, lo, lo + 40)
        T_ref = ap.ap_last_launch()["t_ref"]
        if o["T"] > T_ref:
            assert key == (1 << 63) - 1
        else:
            res = ap.ap_decode(plan, 0, wl.p, wl.m, 1, 8, key=key)
            assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])


def test_fake_sharding_equals_single(ap, oracle_mod):
    """G shards run one after another and min-reduced == the 1-shard key, for
    several G (the multi-GPU decomposition of SURVEY §8e, on one GPU)."""
    wl = synth.config(2)
    f, b, a = wl.arrays()
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    from paper_conf_cluster_liulldgl22_b200.search import shard
    N = ap.ap_count(wl.n, wl.p)
    full = _search(ap, plan, wl.p, wl.m, wl.k_lo, wl.k_hi)
    for G in (2, 3, 8, 13):
        keys = []
        for g in range(G):
            lo, hi = shard(N, g, G)
            keys.append(_search(ap, plan, wl.p, wl.m, wl.k_lo, wl.k_hi, lo, hi))
        assert min(keys) == full


# --------------------------------------------------------------------------- K3
def test_heuristic_random_vs_oracle(ap, oracle_mod):
    rng = np.random.default_rng(8)
    import torch
    for trial in range(10):
        n = int(rng.integers(6, 30))
        f, b, a = synth.random_tables(trial, n, ["b3f", "uniform", "small"][trial % 3])
        bw = synth.LINK_BYTES_PER_S if trial % 3 != 2 else 10**9
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        p = int(rng.integers(2, min(n, 9) + 1))
        m = int(rng.integers(1, 3 * p))
        R = 300
        key = torch.empty(1, dtype=torch.int64, device="cuda")
        ap.ap_search_heuristic(plan, p, m, 0x5EED, 2, 0, R, 0, key)
        torch.cuda.synchronize()
        kv = int(key.item())
        o = M.heuristic(p, m, 0x5EED, 2, 0, R)
        assert (kv >> 20, kv & ((1 << 20) - 1)) == (o["T"], o["restart"]), (n, p, m)
        res = ap.ap_decode(plan, 1, p, m, seed=0x5EED, radius=2, key=kv)
        assert res["cuts"] == [int(x) for x in o["cuts"]] and res["time_ns"] == o["T"]
        # per-restart: single-restart ranges give each restart's own T
        for r in (0, 1, 7):
            ap.ap_search_heuristic(plan, p, m, 0x5EED, 2, r, r + 1, 0, key)
            torch.cuda.synchronize()
            assert int(key.item()) >> 20 == M.heuristic_restart(p, m, 0x5EED, 2, r)["T"]


def test_heuristic_C2_and_C5(ap, oracle_mod):
    """C5 at full size: all 65 536 restarts, GPU winner == oracle winner (the oracle
    runs the same restarts on the host cores)."""
    import torch
    for cfg, R in ((2, 4096), (5, 65536)):
        wl = synth.config(cfg)
        f, b, a = wl.arrays()
        M = oracle_mod.Model.from_workload(wl)
        plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
        key = torch.empty(1, dtype=torch.int64, device="cuda")
        ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 0, key)
        torch.cuda.synchronize()
        kv = int(key.item())
        o = M.heuristic_parallel(wl.p, wl.m, wl.seed, wl.radius, 0, R)
        assert (kv >> 20, kv & ((1 << 20) - 1)) == (o["T"], o["restart"])
        res = ap.ap_decode(plan, 1, wl.p, wl.m, seed=wl.seed, radius=wl.radius, key=kv)
        assert res["cuts"] == [int(x) for x in o["cuts"]]
        if cfg == 5:
            assert o["T"] <= 430480412  # restart 0 alone reaches this


# --------------------------------------------------------------------------- slicer
def test_slice_sweep_vs_oracle(ap, oracle_mod):
    for cfg in (1, 2, 4, 5):
        wl = synth.config(cfg)
        f, b, a = wl.arrays()
        M = oracle_mod.Model.from_workload(wl)
        plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
        cuts, _ = M.alg1(wl.p)
        T, bk = ap.ap_slice_sweep(plan, wl.p, wl.m, cuts, 16)
        oT, obk = M.slice_sweep(wl.p, wl.m, cuts, 16)
        assert list(T) == list(oT) and bk == obk


def test_overflow_guard_and_errors(ap):
    import torch
    big = np.full(4, 1 << 58, np.int64)
    plan = ap.ap_plan_create(big, big, np.zeros(4, np.int64), 10**9)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    with pytest.raises(ap.APError) as ei:
        ap.ap_search_exhaustive(plan, 2, 64, 1, 1, 0, 3, key)
    assert ei.value.status == 2
    f, b, a = synth.random_tables(1, 10)
    plan = _plan(ap, f, b, a, synth.LINK_BYTES_PER_S)
    with pytest.raises(ap.APError) as ei:
        ap.ap_search_exhaustive(plan, 4, 8, 1, 1, 5, 5, key)
    assert ei.value.status == 1
    with pytest.raises(ap.APError):
        ap.ap_search_exhaustive(plan, 11, 8, 1, 1, 0, 1, key)
    with pytest.raises(ap.APError):
        ap.ap_decode(plan, 0, 4, 8, 1, 1, key=(1 << 63) - 1)


def test_exhaustive_u32_tight_bound_saturates(ap, oracle_mod, monkeypatch):
    """Large costs so that S = T_ref+1 is near 2^30 and the host's no-wrap bound
    allows only a few rows between clamps: most candidates saturate, the argmin
    must still equal the oracle's and the int64 sweep's key bit for bit."""
    rng = np.random.default_rng(21)
    hits = 0
    for trial in range(16):
        n = int(rng.integers(8, 14))
        p = int(rng.integers(3, 6))
        m = int(rng.integers(p + 8, p + 20))
        # per-row growth W ~ 2^32 / (p + 3 + (m+p)/p): T_ref ~ (m+p) W / p leaves room
        # for only ~p+3 rows between clamps (host bound), so clamps and saturation fire
        hi = int(2 ** 32 / (n * (p + 3 + (m + p) / p)) / 1.25)
        f = rng.integers(hi // 4, hi, n).astype(np.int64)
        b = rng.integers(hi // 4, hi, n).astype(np.int64)
        a = rng.integers(0, 1 << 20, n).astype(np.int64)
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        plan = _plan(ap, f, b, a, synth.LINK_BYTES_PER_S)
        k_hi = int(rng.integers(1, 4))
        monkeypatch.delenv("AP_SWEEP", raising=False)
        key = _search(ap, plan, p, m, 1, k_hi)
        info = ap.ap_last_launch()
        monkeypatch.setenv("AP_SWEEP", "int64")
        key64 = _search(ap, plan, p, m, 1, k_hi)
        assert key == key64
        o = M.exhaustive(p, m, 1, k_hi)
        res = ap.ap_decode(plan, 0, p, m, 1, k_hi, key=key)
        assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])
        # a schedule with more than one clamp inside the steady rows
        if info["fast_u32"] and info["clamp_first"] + info["clamp_rows"] < m - p:
            hits += 1
    assert hits >= 3


def test_exhaustive_u32_clamp_schedules(ap, oracle_mod, monkeypatch):
    """The host's saturating-clamp schedule (no clamp / one clamp /
    clamp right after the warm-up / a final clamp before the cool-down): over cost
    scales that produce every schedule, the u32
    key equals the int64 sweep's and the oracle's argmin, in all three search modes."""
    rng = np.random.default_rng(77)
    seen = set()
    for trial in range(40):
        n = int(rng.integers(9, 13))
        p = int(rng.choice([3, 4, 5, 8]))
        p = min(p, n - 1)
        m = int(rng.integers(p, p + 40))
        scale = float(2.0 ** rng.uniform(10, 26))
        f = (rng.uniform(0.3, 1.0, n) * scale).astype(np.int64)
        b = (rng.uniform(0.3, 1.0, n) * 3 * scale).astype(np.int64)
        a = rng.integers(0, 1 << 22, n).astype(np.int64)
        plan = _plan(ap, f, b, a, synth.LINK_BYTES_PER_S)
        k_hi = int(rng.integers(1, 4))
        monkeypatch.delenv("AP_SWEEP", raising=False)
        key = _search(ap, plan, p, m, 1, k_hi)
        info = ap.ap_last_launch()
        keys = [_search_mode(ap, plan, p, m, 1, k_hi, md) for md in (1, 2)]
        monkeypatch.setenv("AP_SWEEP", "int64")
        key64 = _search(ap, plan, p, m, 1, k_hi)
        assert key == key64 == keys[0] == keys[1], (trial, info)
        if info["fast_u32"]:
            steady = m - p
            if info["clamp_first"] > steady:
                kind = "none"
            elif info["clamp_first"] == 0:
                kind = "after-warmup"
            else:
                kind = "first-segment"
            seen.add(kind)
            if info["clamp_final"]:
                seen.add("final")
            if trial % 4 == 0:
                M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
                o = M.exhaustive(p, m, 1, k_hi)
                res = ap.ap_decode(plan, 0, p, m, 1, k_hi, key=key)
                assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])
    assert {"none", "first-segment", "final"} <= seen, seen


def test_key_layout_matches_python_helpers(ap):
    """The C key layout == search.pack/unpack (used by the multi-process host logic)."""
    from paper_conf_cluster_liulldgl22_b200.search import unpack_exhaustive_key
    wl = synth.config(2)
    f, b, a = wl.arrays()
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    key = _search(ap, plan, wl.p, wl.m, wl.k_lo, wl.k_hi)
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=key)
    assert unpack_exhaustive_key(key, N, wl.k_lo, wl.k_hi) == (res["time_ns"], res["rank"], res["k"])


def test_heuristic_sims_count_matches_oracle(ap, oracle_mod):
    """ap_last_sims after a heuristic search == the oracle's simulation count for the
    same restarts (start partition + every non-duplicate child)."""
    import torch
    for cfg, R in ((2, 512), (5, 256)):
        wl = synth.config(cfg)
        f, b, a = wl.arrays()
        plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
        key = torch.empty(1, dtype=torch.int64, device="cuda")
        ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 0, key)
        torch.cuda.synchronize()
        o = oracle_mod.Model.from_workload(wl).heuristic(wl.p, wl.m, wl.seed, wl.radius, 0, R)
        assert ap.ap_last_sims() == o["sims"]
        if cfg == 2:
            ap.ap_search_exhaustive(plan, wl.p, wl.m, 1, 2, 0, 1000, key)
            assert ap.ap_last_sims() == 1000 * 2


def _search_mode(ap, plan, p, m, k_lo, k_hi, mode, lo=None, hi=None):
    import torch
    N = ap.ap_count(plan.n, p)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_search_exhaustive_mode(plan, p, m, k_lo, k_hi, 0 if lo is None else lo,
                                 N if hi is None else hi, mode, key)
    torch.cuda.synchronize()
    return int(key.item())


def test_search_modes_equal_random(ap, oracle_mod):
    """k-factored and pruned modes return exactly the full sweep's key (and the
    oracle's argmin) on random problems, incl. saturating near-2^32 tables."""
    rng = np.random.default_rng(31)
    for trial in range(24):
        n = int(rng.integers(4, 16))
        p = int(rng.integers(2, min(n, 8) + 1))
        m = int(rng.integers(p, p + 12))
        if trial % 3 == 2:
            hi = int(2 ** 32 / (n * (p + 3 + (m + p) / p)) / 1.25)
            f = rng.integers(hi // 4, hi, n).astype(np.int64)
            b = rng.integers(hi // 4, hi, n).astype(np.int64)
            a = rng.integers(0, 1 << 20, n).astype(np.int64)
            bw = synth.LINK_BYTES_PER_S
        else:
            kind = ["uniform", "b3f", "small"][trial % 3]
            f, b, a = synth.random_tables(trial, n, kind)
            bw = synth.link_for(kind)
        plan = _plan(ap, f, b, a, bw)
        k_lo = int(rng.integers(1, 3)); k_hi = k_lo + int(rng.integers(0, 6))
        keys = [_search_mode(ap, plan, p, m, k_lo, k_hi, mode) for mode in (0, 1, 2)]
        assert keys[0] == keys[1] == keys[2], (n, p, m, k_lo, k_hi, keys)
        o = oracle_mod.Model(f, b, a, bw).exhaustive(p, m, k_lo, k_hi)
        res = ap.ap_decode(plan, 0, p, m, k_lo, k_hi, key=keys[1])
        assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])


@pytest.mark.parametrize("cfg", [2, 3, 4])
def test_search_modes_equal_configs(ap, cfg):
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    keys = [_search_mode(ap, plan, wl.p, wl.m, wl.k_lo, wl.k_hi, mode) for mode in (0, 1, 2)]
    assert keys[0] == keys[1] == keys[2]
    if cfg == 4:
        # sampled windows too (the k-factored path on arbitrary slices)
        N = ap.ap_count(wl.n, wl.p)
        for lo in (0, N // 3, N - 5000):
            ks = [_search_mode(ap, plan, wl.p, wl.m, 1, 8, mode, lo, lo + 5000) for mode in (0, 1, 2)]
            assert ks[0] == ks[1] == ks[2]


@pytest.mark.parametrize("mode", ["", "int64", "redo"])
def test_heuristic_fast_and_redo_paths(ap, oracle_mod, monkeypatch, mode):
    """The u32 restart kernel, the exact int64 kernel, and the u32 kernel with a bound
    so low that many restarts saturate and are redone exactly, all give the oracle's
    winner and simulation count (C2, p=4: the fast path applies)."""
    import torch
    wl = synth.config(2)
    f, b, a = wl.arrays()
    M = oracle_mod.Model.from_workload(wl)
    R = 1024
    o = M.heuristic(wl.p, wl.m, wl.seed, wl.radius, 0, R, per_restart=True)
    if mode == "int64":
        monkeypatch.setenv("AP_HEUR", "int64")
    if mode == "redo":
        monkeypatch.setenv("AP_HEUR_S", str(int(np.median(o["per_restart_T"]))))
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 0, key)
    torch.cuda.synchronize()
    kv = int(key.item())
    assert (kv >> 20, kv & 0xFFFFF) == (o["T"], o["restart"])
    assert ap.ap_last_sims() == o["sims"]
    res = ap.ap_decode(plan, 1, wl.p, wl.m, seed=wl.seed, radius=wl.radius, key=kv)
    assert res["cuts"] == [int(x) for x in o["cuts"]]


@pytest.mark.parametrize("cfg,R", [(2, 512), (3, 256), (5, 1024)])
def test_heuristic_adjust_eq1_vs_oracle(ap, oracle_mod, cfg, R):
    """adjust_mode 1 (paper step 2, Eq. (1)): GPU winner, decode and simulation count
    equal the oracle's walk with the same reading (Q19)."""
    import torch
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    M = oracle_mod.Model.from_workload(wl)
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 1, key)
    torch.cuda.synchronize()
    kv = int(key.item())
    o = M.heuristic_parallel(wl.p, wl.m, wl.seed, wl.radius, 0, R, adjust_mode=1)
    assert (kv >> 20, kv & 0xFFFFF) == (o["T"], o["restart"])
    assert ap.ap_last_sims() == o["sims"]
    res = ap.ap_decode(plan, 1, wl.p, wl.m, seed=wl.seed, radius=wl.radius, adjust_mode=1, key=kv)
    assert res["cuts"] == [int(x) for x in o["cuts"]]


def test_heuristic_adjust_eq1_random(ap, oracle_mod):
    import torch
    rng = np.random.default_rng(77)
    for trial in range(8):
        n = int(rng.integers(8, 30))
        f, b, a = synth.random_tables(trial + 50, n, ["b3f", "uniform"][trial % 2])
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        plan = _plan(ap, f, b, a, synth.LINK_BYTES_PER_S)
        p = int(rng.choice([3, 4, 5, 8]))
        if p > n:
            continue
        m = int(rng.integers(1, 3 * p))
        key = torch.empty(1, dtype=torch.int64, device="cuda")
        ap.ap_search_heuristic(plan, p, m, 0x5EED, 2, 0, 200, 1, key)
        torch.cuda.synchronize()
        kv = int(key.item())
        o = M.heuristic(p, m, 0x5EED, 2, 0, 200, adjust_mode=1)
        assert (kv >> 20, kv & 0xFFFFF) == (o["T"], o["restart"]), (n, p, m)
        assert ap.ap_last_sims() == o["sims"]


def test_slice_sweep_paper_vs_oracle(ap, oracle_mod):
    """Paper Slicer form on the GPU (generic sim with s sliced micro-batches) == oracle,
    incl. m < p-1, k = 2..4, every s in [0, m]."""
    rng = np.random.default_rng(41)
    for trial in range(25):
        kind = ["uniform", "b3f", "small"][trial % 3]
        n = int(rng.integers(2, 25))
        f, b, a = synth.random_tables(trial, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        p = int(rng.integers(1, min(n, 16) + 1))
        m = int(rng.integers(1, 2 * p + 4))
        k = int(rng.integers(2, 5))
        cuts = synth.random_cuts(trial, n, p, 1)[0]
        T, bs = ap.ap_slice_sweep_paper(plan, p, m, cuts, k, m)
        oT, obs = M.slice_sweep_paper(p, m, cuts, k, m)
        assert list(T) == list(oT) and bs == obs, (n, p, m, k)
    for cfg in synth.ALL_CONFIGS:
        wl = synth.config(cfg)
        f, b, a = wl.arrays()
        M = oracle_mod.Model.from_workload(wl)
        plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
        c, _ = M.alg1(wl.p)
        T, bs = ap.ap_slice_sweep_paper(plan, wl.p, wl.m, c, 2, wl.p)
        oT, obs = M.slice_sweep_paper(wl.p, wl.m, c, 2, wl.p)
        assert list(T) == list(oT) and bs == obs
        for rd in (0, 1):
            assert ap.ap_slicer_alg2(plan, wl.p, c, rd) == M.alg2(wl.p, c, rd)


def test_alg2_random_vs_oracle(ap, oracle_mod):
    rng = np.random.default_rng(43)
    for trial in range(30):
        n = int(rng.integers(2, 40))
        f, b, a = synth.random_tables(trial, n, ["uniform", "b3f", "small"][trial % 3])
        M = oracle_mod.Model(f, b, a, synth.LINK_BYTES_PER_S)
        plan = _plan(ap, f, b, a, synth.LINK_BYTES_PER_S)
        p = int(rng.integers(1, min(n, 32) + 1))
        cuts = synth.random_cuts(trial, n, p, 1)[0]
        for rd in (0, 1):
            assert ap.ap_slicer_alg2(plan, p, cuts, rd) == M.alg2(p, cuts, rd), (n, p, rd)


# --------------------------------------------------------------------------- N3 minLB
def test_min_lower_bound_vs_oracle(ap, oracle_mod):
    """ap_min_lower_bound: bit-exact value and argmin cuts vs the oracle's DP, over
    table kinds, p up to 32, K up to 16, n up to 512 (the AP_MAX_N edge)."""
    rng = np.random.default_rng(14)
    cases = [(int(rng.integers(1, 60)), kind) for kind in
             ["uniform", "b3f", "small", "equal", "huge", "zero"] for _ in range(6)]
    cases += [(512, "uniform"), (512, "b3f"), (1, "uniform"), (2, "small")]
    for i, (n, kind) in enumerate(cases):
        f, b, a = synth.random_tables(1000 + i, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        for p in sorted({1, min(n, 2), int(rng.integers(1, min(n, 32) + 1)), min(n, 32)}):
            m = int(rng.choice([1, 2, p, 4 * p + 1, 64]))
            K = int(rng.integers(1, 17))
            lb, cuts = ap.ap_min_lower_bound(plan, p, m, K)
            olb, ocuts = M.min_lower_bound(p, m, K)
            assert lb == olb, (n, kind, p, m, K)
            assert list(cuts) == list(ocuts), (n, kind, p, m, K)


@pytest.mark.parametrize("cfg", [1, 2, 3, 4, 5])
def test_min_lower_bound_configs(ap, oracle_mod, cfg):
    """Configs: GPU == oracle, and the bound never exceeds a GPU-found plan's T."""
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    M = oracle_mod.Model.from_workload(wl)
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    K = wl.k_hi if cfg != 5 else 1
    lb, cuts = ap.ap_min_lower_bound(plan, wl.p, wl.m, K)
    assert (lb, list(cuts)) == (lambda r: (r[0], list(r[1])))(M.min_lower_bound(wl.p, wl.m, K))
    c1, _ = ap.ap_alg1(plan, wl.p)
    assert lb <= M.T(wl.p, wl.m, c1, k=1)


def test_min_lower_bound_errors(ap):
    f, b, a = synth.random_tables(3, 10, "uniform")
    plan = _plan(ap, f, b, a, synth.link_for("uniform"))
    for args in [(0, 4, 1), (11, 4, 1), (3, 0, 1), (3, 4, 0), (3, 4, 17)]:
        with pytest.raises(ap.APError):
            ap.ap_min_lower_bound(plan, *args)


# --------------------------------------------------------------------------- N3 two-phase
def _search2(ap, plan, p, m, k_lo, k_hi, mode=0, lo=None, hi=None):
    import torch
    N = ap.ap_count(plan.n, p)
    out = torch.empty(2, dtype=torch.int64, device="cuda")
    ap.ap_search_exhaustive2(plan, p, m, k_lo, k_hi, 0 if lo is None else lo,
                             N if hi is None else hi, mode, out)
    torch.cuda.synchronize()
    return int(out[0].item()), int(out[1].item())


@pytest.mark.parametrize("sweep", ["", "int64", "generic"])
def test_two_phase_vs_oracle_random(ap, oracle_mod, sweep, monkeypatch):
    """ap_search_exhaustive2 + ap_decode mode 2 == oracle argmin (T, rank, k), every
    search mode, and == the packed key wherever that fits."""
    if sweep:
        monkeypatch.setenv("AP_SWEEP", sweep)
    rng = np.random.default_rng(23)
    for trial in range(12):
        kind = ["uniform", "b3f", "small", "equal"][trial % 4]
        n = int(rng.integers(3, 18))
        f, b, a = synth.random_tables(300 + trial, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        p = int(rng.integers(1, min(n, 8) + 1))
        m = int(rng.choice([1, 2, p, p + 3, 12]))
        k_lo = int(rng.integers(1, 3)); k_hi = k_lo + int(rng.integers(0, 4))
        K = k_hi - k_lo + 1
        o = M.exhaustive(p, m, k_lo, k_hi)
        packed = _search(ap, plan, p, m, k_lo, k_hi)
        for mode in (0, 1, 2):
            T, idx = _search2(ap, plan, p, m, k_lo, k_hi, mode)
            assert (T, idx // K, k_lo + idx % K) == (o["T"], o["rank"], o["k"]), (trial, mode)
            res = ap.ap_decode(plan, 2, p, m, k_lo, k_hi, key=idx)
            assert res["time_ns"] == T and res["cuts"] == [int(x) for x in o["cuts"]]
            from paper_conf_cluster_liulldgl22_b200.search import rank_bits
            assert packed == (T << rank_bits(ap.ap_count(n, p), K)) | idx


def test_two_phase_when_packed_key_does_not_fit(ap, oracle_mod):
    """T ~ 2^51 with rb = 14: the packed key is RANGE; the two-phase search (and the
    search_exhaustive orchestration that falls back to it) returns the oracle argmin."""
    import torch
    from paper_conf_cluster_liulldgl22_b200.search import search_exhaustive, shard
    for seed in range(3):
        f, b, a = synth.random_tables(40 + seed, 30, "uniform", fmax=1 << 44)
        bw = synth.link_for("uniform")
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        p, m, k_lo, k_hi = 4, 16, 1, 4
        key = torch.empty(1, dtype=torch.int64, device="cuda")
        # the packing test needs T_ref (device-side): the key comes back as AP_KEY_RANGE,
        # and decoding it is the RANGE error
        ap.ap_search_exhaustive(plan, p, m, k_lo, k_hi, 0, ap.ap_count(30, p), key)
        torch.cuda.synchronize()
        assert int(key.item()) == ap.AP_KEY_RANGE
        with pytest.raises(ap.APError) as ei:
            ap.ap_decode(plan, 0, p, m, k_lo, k_hi, key=int(key.item()))
        assert ei.value.status == ap.AP_ERR_RANGE
        o = M.exhaustive(p, m, k_lo, k_hi)
        assert o["T"] >= 1 << 48
        for mode in (0, 1, 2):
            T, idx = _search2(ap, plan, p, m, k_lo, k_hi, mode)
            assert (T, idx // 4, 1 + idx % 4) == (o["T"], o["rank"], o["k"])
        r = search_exhaustive(plan, p, m, k_lo, k_hi)
        assert r["two_phase"] and (r["time_ns"], r["rank"], r["k"]) == (o["T"], o["rank"], o["k"])
        assert r["cuts"] == [int(x) for x in o["cuts"]]
        # G shards on one GPU combined with the device phase-2 select
        N = ap.ap_count(30, p)
        for G in (2, 5):
            locs = [torch.tensor(_search2(ap, plan, p, m, k_lo, k_hi, 0, *shard(N, g, G)),
                                 dtype=torch.int64, device="cuda") for g in range(G)]
            t_star = torch.tensor([min(int(l[0]) for l in locs)], dtype=torch.int64, device="cuda")
            idxs = []
            for l in locs:
                idx = torch.empty(1, dtype=torch.int64, device="cuda")
                ap.ap_key2_select(l, t_star, idx)
                idxs.append(int(idx.item()))
            assert (int(t_star.item()), min(idxs)) == (o["T"], o["rank"] * 4 + o["k"] - 1)


@pytest.mark.parametrize("cfg", [2, 3])
def test_two_phase_configs_match_packed(ap, cfg):
    """On the configs (where the packed key fits) both reductions pick the same plan."""
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    K = wl.k_hi - wl.k_lo + 1
    from paper_conf_cluster_liulldgl22_b200.search import rank_bits
    key = _search(ap, plan, wl.p, wl.m, wl.k_lo, wl.k_hi)
    T, idx = _search2(ap, plan, wl.p, wl.m, wl.k_lo, wl.k_hi)
    assert key == (T << rank_bits(N, K)) | idx


# --------------------------------------------------------------------------- N1 reach
def _reach(ap, plan, p, m, seed, radius, r_lo, r_hi, vmax):
    import torch
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_search_reachable(plan, p, m, seed, radius, r_lo, r_hi, vmax, key)
    torch.cuda.synchronize()
    return int(key.item()), ap.ap_last_sims(), ap.ap_last_truncated()


def test_reach_random_vs_oracle(ap, oracle_mod):
    """ap_search_reachable == oracle or_reach: winner (T, restart), decoded cuts, total
    simulations and truncated-restart count -- including tiny vmax (truncation)."""
    rng = np.random.default_rng(31)
    for trial in range(16):
        kind = ["uniform", "b3f", "small", "equal"][trial % 4]
        n = int(rng.integers(4, 60))
        f, b, a = synth.random_tables(500 + trial, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        p = int(rng.integers(1, min(n, 20) + 1))
        m = int(rng.choice([1, 2, p, p + 3, 24]))
        seed, radius = int(rng.integers(0, 1 << 30)), int(rng.integers(0, 4))
        R = int(rng.integers(1, 200))
        vmax = int(rng.choice([1, 3, 8, 1024]))
        key, sims, trunc = _reach(ap, plan, p, m, seed, radius, 0, R, vmax)
        o = M.reach(p, m, seed, radius, 0, R, vmax=vmax)
        assert (key >> 20, key & 0xFFFFF) == (o["T"], o["restart"]), (trial, n, p, m, vmax)
        assert (sims, trunc) == (o["sims"], o["truncated"]), (trial, n, p, m, vmax)
        res = ap.ap_decode_reachable(plan, p, m, seed, radius, vmax, key)
        assert res["time_ns"] == o["T"] and res["cuts"] == [int(x) for x in o["cuts"]]
        assert res["master"] == M.simulate(p, m, o["cuts"])["master"]


@pytest.mark.parametrize("cfg,R", [(2, 1024), (3, 512), (4, 256), (5, 2048)])
def test_reach_configs_vs_oracle(ap, oracle_mod, cfg, R):
    """Configs: same winner, simulations and truncations as the oracle, and never
    worse than the greedy walk over the same restarts."""
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    M = oracle_mod.Model.from_workload(wl)
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    key, sims, trunc = _reach(ap, plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 1024)
    o = M.reach_parallel(wl.p, wl.m, wl.seed, wl.radius, 0, R, vmax=1024)
    assert (key >> 20, key & 0xFFFFF, sims, trunc) == (o["T"], o["restart"], o["sims"], o["truncated"])
    import torch
    hk = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 0, hk)
    torch.cuda.synchronize()
    assert key >> 20 <= int(hk.item()) >> 20


def test_reach_errors(ap):
    import torch
    f, b, a = synth.random_tables(3, 10, "uniform")
    plan = _plan(ap, f, b, a, synth.link_for("uniform"))
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    for args in [(3, 4, 0, 2, 5, 5, 8), (3, 4, 0, 2, 0, 8, 0), (3, 4, 0, -1, 0, 8, 8),
                 (3, 4, 0, 2, 0, (1 << 20) + 1, 8)]:
        with pytest.raises(ap.APError):
            ap.ap_search_reachable(plan, *args, key)


# --------------------------------------------------------------------------- N4 depth
def test_memory_mode_random_vs_oracle(ap, oracle_mod):
    """AP_SEARCH_MEMORY == the oracle's feasible argmin (T, rank, k), with capacities
    from 'nothing fits' to 'everything fits', including an infeasible Alg.-1 start
    (search_exhaustive's two-phase fallback)."""
    from paper_conf_cluster_liulldgl22_b200.search import search_exhaustive
    rng = np.random.default_rng(44)
    for trial in range(14):
        kind = ["uniform", "b3f", "small", "equal"][trial % 4]
        n = int(rng.integers(3, 16))
        f, b, a = synth.random_tables(700 + trial, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        st = rng.integers(0, 1 << 30, n)
        sh = rng.integers(0, 1 << 26, n)
        p = int(rng.integers(1, min(n, 6) + 1))
        m = int(rng.choice([1, 2, p, p + 3, 12]))
        k_hi = int(rng.integers(1, 4))
        tot = int(st.sum() + min(p, m) * sh.sum())
        for cap in (tot // 8, tot // 3, tot // 2, tot):
            ap.ap_plan_set_memory(plan, st, sh, cap)
            r = search_exhaustive(plan, p, m, 1, k_hi, mode=ap.AP_SEARCH_MEMORY)
            o = M.exhaustive_mem(p, m, 1, k_hi, st, sh, cap)
            if o["T"] is None:
                assert r["key"] == ap.INT64_MAX, (trial, cap)
                continue
            assert (r["time_ns"], r["rank"], r["k"]) == (o["T"], o["rank"], o["k"]), (trial, cap)


def test_plan_pipeline_depth_vs_oracle(ap, oracle_mod):
    """The N4 workload (GPT-2 1.3B, mbs 16, 8 GPUs, 24 GiB): every depth's feasible
    argmin and the chosen depth equal the oracle's (p = 8 on sampled rank windows)."""
    import torch
    from paper_conf_cluster_liulldgl22_b200.search import plan_pipeline_depth
    d = synth.depth_config()
    f, b, a = d.base.arrays()
    plan = _plan(ap, f, b, a, d.base.link_bytes_per_s)
    ap.ap_plan_set_memory(plan, d.static_bytes, d.stash_bytes, d.cap_bytes)
    M = oracle_mod.Model.from_workload(d.base)
    out = plan_pipeline_depth(plan, d.n_gpus, d.microbatches)
    rows = {r["p"]: r for r in out["per_depth"]}
    assert sorted(rows) == [1, 2, 4, 8]
    for p in (1, 2, 4):
        o = M.exhaustive_mem(p, rows[p]["m"], 1, 1, d.static_bytes, d.stash_bytes, d.cap_bytes)
        assert rows[p]["T"] == o["T"]
        if o["T"] is not None:
            assert (rows[p]["rank"], rows[p]["cuts"]) == (o["rank"], [int(x) for x in o["cuts"]])
    feas = [(rows[p]["T"], p) for p in rows if rows[p]["T"] is not None]
    assert out["best"]["p"] == min(feas)[1]
    # p = 8 on windows: the device feasible argmin of [lo, hi) == the oracle's
    N = ap.ap_count(d.base.n, 8)
    m8 = rows[8]["m"]
    out2 = torch.empty(2, dtype=torch.int64, device="cuda")
    # a shard keeps only candidates with T <= T_ref (the Alg.-1 partition's T when it
    # fits; include/ap.h AP_SEARCH_MEMORY)
    a1, _ = M.alg1(8)
    tref = (M.T(8, m8, a1) if M.feasible(8, m8, a1, d.static_bytes, d.stash_bytes, d.cap_bytes)
            else None)
    r1 = oracle_mod.rank(d.base.n, 8, a1)
    nontrivial = 0
    for lo in (0, N // 3, N - 20000, max(0, r1 - 10000)):
        hi = lo + 20000
        ap.ap_search_exhaustive2(plan, 8, m8, 1, 1, lo, hi, ap.AP_SEARCH_MEMORY, out2)
        torch.cuda.synchronize()
        o = M.exhaustive_mem(8, m8, 1, 1, d.static_bytes, d.stash_bytes, d.cap_bytes, lo, hi)
        if o["T"] is None or (tref is not None and o["T"] > tref):
            assert int(out2[0]) == ap.INT64_MAX
        else:
            assert (int(out2[0]), int(out2[1])) == (o["T"], o["rank"])
            nontrivial += 1
    assert nontrivial >= 1


def test_memory_mode_errors(ap):
    import torch
    f, b, a = synth.random_tables(3, 10, "uniform")
    plan = _plan(ap, f, b, a, synth.link_for("uniform"))
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    with pytest.raises(ap.APError):  # no memory model yet
        ap.ap_search_exhaustive_mode(plan, 3, 4, 1, 1, 0, 36, ap.AP_SEARCH_MEMORY, key)
    with pytest.raises(ap.APError):
        ap.ap_plan_set_memory(plan, [-1] * 10, [0] * 10, 100)
    with pytest.raises(ap.APError):
        ap.ap_plan_set_memory(plan, [1 << 61] * 10, [0] * 10, 100)


@pytest.mark.parametrize("p", [2, 4, 8, 16])
def test_heuristic_pool_vs_lane_kernel_and_oracle(ap, oracle_mod, monkeypatch, p):
    """The per-CTA simulation-pool restart kernel (k_heur_pool) and the
    lane-per-restart kernel (AP_HEUR_POOL=0) give the oracle's winner and simulation
    count, and every restart's own best scheme (read back through decode's per-restart
    cache) equals the oracle's replay of that restart."""
    import torch
    rng = np.random.default_rng(100 + p)
    n = int(rng.integers(max(p + 4, 2 * p), 3 * p + 20))
    f, b, a = synth.random_tables(p, n, "b3f")
    bw = synth.LINK_BYTES_PER_S
    m = int(rng.integers(p, 3 * p + 2))
    R = 3000
    M = oracle_mod.Model(f, b, a, bw)
    o = M.heuristic_parallel(p, m, 0x5EED, 2, 0, R, per_restart=True)
    plan = _plan(ap, f, b, a, bw)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    for pool in ("1", "0"):
        monkeypatch.setenv("AP_HEUR_POOL", pool)
        ap.ap_search_heuristic(plan, p, m, 0x5EED, 2, 0, R, 0, key)
        torch.cuda.synchronize()
        kv = int(key.item())
        assert (kv >> 20, kv & 0xFFFFF) == (o["T"], o["restart"]), (pool, n, p, m)
        assert ap.ap_last_sims() == o["sims"], pool
        for r in [0, 1, 2, R // 2, R - 1] + [int(x) for x in rng.integers(0, R, 5)]:
            k_r = (int(o["per_restart_T"][r]) << 20) | r
            res = ap.ap_decode(plan, 1, p, m, seed=0x5EED, radius=2, key=k_r)
            want = M.heuristic_restart(p, m, 0x5EED, 2, r)
            assert res["time_ns"] == want["T"] and res["cuts"] == [int(x) for x in want["cuts"]], (pool, r)


def test_exhaustive_div1_pieces(ap, oracle_mod, monkeypatch):
    """The one-umulhi floor(v/k) of the slice pieces (values < 2^28) and the corrected
    two-step form (AP_DIV1=0) give the same key as the oracle's argmin, on C2 (k 1..4)
    and on random tables with values just below the 2^28 bound."""
    import torch
    cases = []
    wl = synth.config(2)
    cases.append((*wl.arrays(), wl.link_bytes_per_s, wl.p, wl.m, 1, 4))
    rng = np.random.default_rng(77)
    for t in range(4):
        n = int(rng.integers(6, 12))
        f = rng.integers((1 << 28) // (2 * n), (1 << 28) // n, n).astype(np.int64)
        b = rng.integers(0, 1 << 20, n).astype(np.int64)
        a = rng.integers(0, 1 << 27, n).astype(np.int64)
        p = int(rng.integers(2, min(n, 8) + 1))
        cases.append((f, b, a, 10**9, p, int(rng.integers(p, p + 6)), 1, 16))
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    for f, b, a, bw, p, m, k_lo, k_hi in cases:
        plan = _plan(ap, f, b, a, bw)
        N = ap.ap_count(len(f), p)
        keys = []
        for d in ("1", "0"):
            monkeypatch.setenv("AP_DIV1", d)
            ap.ap_search_exhaustive(plan, p, m, k_lo, k_hi, 0, N, key)
            torch.cuda.synchronize()
            keys.append(int(key.item()))
        assert keys[0] == keys[1]
        o = oracle_mod.Model(f, b, a, bw).exhaustive(p, m, k_lo, k_hi)
        res = ap.ap_decode(plan, 0, p, m, k_lo, k_hi, key=keys[0])
        assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])


@pytest.mark.parametrize("mode", ["fast", "int64", "saturating"])
def test_reach_fast_and_exact_simulation(ap, oracle_mod, monkeypatch, mode):
    """The reachable-set kernel's u32 fast simulation (p in {2,4,8,16}, m >= p), the
    exact int64 one (AP_HEUR=int64) and the fast one with a bound so low that many
    simulations fall back to int64 (AP_HEUR_S) all give the oracle's winner,
    simulation count and truncations."""
    if mode == "int64":
        monkeypatch.setenv("AP_HEUR", "int64")
    rng = np.random.default_rng(61)
    for trial, p in enumerate((2, 4, 8, 16)):
        n = int(rng.integers(p + 6, 3 * p + 20))
        f, b, a = synth.random_tables(900 + trial, n, "b3f")
        bw = synth.LINK_BYTES_PER_S
        M = oracle_mod.Model(f, b, a, bw)
        m = int(rng.integers(p, 3 * p + 2))
        R = 300
        o = M.reach_parallel(p, m, 0x5EED, 2, 0, R, vmax=1024)
        if mode == "saturating":
            monkeypatch.setenv("AP_HEUR_S", str(int(o["T"]) + 1))
        plan = _plan(ap, f, b, a, bw)
        key, sims, trunc = _reach(ap, plan, p, m, 0x5EED, 2, 0, R, 1024)
        assert (key >> 20, key & 0xFFFFF, sims, trunc) == (o["T"], o["restart"], o["sims"], o["truncated"]), (mode, p)
        res = ap.ap_decode_reachable(plan, p, m, 0x5EED, 2, 1024, key)
        assert res["time_ns"] == o["T"] and res["cuts"] == [int(x) for x in o["cuts"]]


@pytest.mark.parametrize("pool", ["1", "0"])
def test_reach_pool_and_quad_kernels(ap, oracle_mod, monkeypatch, pool):
    """Both reachable-set kernels -- the simulation pool (default) and the 4-lane-group
    kernel (AP_REACH_POOL=0; also used for vmax > 2048 and the decode replay) -- give
    the oracle's winner, simulation count and truncations, incl. vmax > 2048."""
    monkeypatch.setenv("AP_REACH_POOL", pool)
    rng = np.random.default_rng(71)
    for trial in range(6):
        n = int(rng.integers(8, 40))
        f, b, a = synth.random_tables(700 + trial, n, ["b3f", "uniform", "equal"][trial % 3])
        bw = synth.link_for(["b3f", "uniform", "equal"][trial % 3])
        M = oracle_mod.Model(f, b, a, bw)
        plan = _plan(ap, f, b, a, bw)
        p = int(rng.choice([2, 3, 4, 8]))
        m = int(rng.integers(1, 3 * p))
        vmax = int(rng.choice([2, 16, 1024, 4096]))
        key, sims, trunc = _reach(ap, plan, p, m, 0x5EED, 2, 0, 150, vmax)
        o = M.reach(p, m, 0x5EED, 2, 0, 150, vmax=vmax)
        assert (key >> 20, key & 0xFFFFF, sims, trunc) == (o["T"], o["restart"], o["sims"], o["truncated"]), (pool, trial)


@pytest.mark.parametrize("mode", ["fast", "int64", "saturating"])
def test_eval_batch_fast_path(ap, oracle_mod, monkeypatch, mode):
    """ap_eval_batch's u32 fast path (p in {2,4,8,16}, m >= p: N-form sweep for T, the
    bit-recording sweep + branch-free backtrack for T + master at k = 1), the exact
    int64 kernel (AP_EVAL=int64) and the fast path with a bound low enough that many
    candidates fall back to int64 (AP_EVAL_S): T and master equal the oracle's for
    every candidate, k up to 16."""
    import torch
    if mode == "int64":
        monkeypatch.setenv("AP_EVAL", "int64")
    rng = np.random.default_rng(83)
    for trial, p in enumerate((2, 4, 8, 16, 8)):
        n = int(rng.integers(p + 2, 3 * p + 20))
        kind = ["b3f", "uniform", "equal", "small", "huge"][trial]
        f, b, a = synth.random_tables(1200 + trial, n, kind)
        bw = synth.link_for(kind)
        M = oracle_mod.Model(f, b, a, bw)
        m = int(rng.integers(p, 3 * p + 3))
        cnt = 64
        cuts = np.sort(np.argsort(rng.random((cnt, n - 1)), axis=1)[:, : p - 1] + 1, axis=1).astype(np.int32)
        ks = rng.integers(1, 17, cnt).astype(np.int32)
        want = [M.simulate(p, m, list(c), k=int(k))["T"] for c, k in zip(cuts, ks)]
        if mode == "saturating":
            monkeypatch.setenv("AP_EVAL_S", str(int(np.median(want))))
        plan = _plan(ap, f, b, a, bw)
        dc = torch.from_numpy(cuts).cuda()
        T = torch.empty(cnt, dtype=torch.int64, device="cuda")
        ap.ap_eval_batch(plan, p, m, dc, torch.from_numpy(ks).cuda(), T)
        torch.cuda.synchronize()
        assert T.tolist() == want, (mode, p, kind)
        k1 = torch.ones(cnt, dtype=torch.int32, device="cuda")
        Mst = torch.empty(cnt, dtype=torch.int32, device="cuda")
        ap.ap_eval_batch(plan, p, m, dc, k1, T, Mst)
        torch.cuda.synchronize()
        o = [M.simulate(p, m, list(c)) for c in cuts]
        assert T.tolist() == [x["T"] for x in o] and Mst.tolist() == [x["master"] for x in o], (mode, p, kind)


def test_pruned_prefix_skips_random_windows(ap, oracle_mod):
    """The pruned mode's prefix jumps (first failing stage bound, and its compute-only
    monotone form) never skip a winner: on random problems and random rank windows the
    key equals the full sweep's and the oracle's argmin over the same window."""
    import torch
    rng = np.random.default_rng(97)
    for trial in range(40):
        n = int(rng.integers(6, 22))
        p = int(rng.integers(2, min(n, 8) + 1))
        m = int(rng.integers(p, p + 10))
        kind = ["b3f", "uniform", "huge", "small"][trial % 4]
        f, b, a = synth.random_tables(1500 + trial, n, kind)
        bw = synth.link_for(kind)
        plan = _plan(ap, f, b, a, bw)
        N = ap.ap_count(n, p)
        lo = int(rng.integers(0, N))
        hi = int(rng.integers(lo + 1, N + 1))
        k_lo = int(rng.integers(1, 3)); k_hi = k_lo + int(rng.integers(0, 4))
        k0 = _search_mode(ap, plan, p, m, k_lo, k_hi, 0, lo, hi)
        k2 = _search_mode(ap, plan, p, m, k_lo, k_hi, 2, lo, hi)
        assert k0 == k2, (trial, n, p, m, lo, hi)
        if k0 != 0x7fffffffffffffff:
            o = oracle_mod.Model(f, b, a, bw).exhaustive(p, m, k_lo, k_hi, lo, hi)
            res = ap.ap_decode(plan, 0, p, m, k_lo, k_hi, key=k0)
            assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])


def test_exhaustive_bounded(ap, oracle_mod):
    """ap_search_exhaustive_bounded: with t_bound = an attained T >= the optimum (the
    heuristic's, or the optimum itself) every mode returns the oracle's argmin; with
    t_bound = optimum - 1 every shard is empty."""
    import torch
    rng = np.random.default_rng(41)
    out = torch.empty(2, dtype=torch.int64, device="cuda")
    hk = torch.empty(1, dtype=torch.int64, device="cuda")
    for trial in range(12):
        n = int(rng.integers(6, 20))
        p = int(rng.integers(2, min(n, 8) + 1))
        m = int(rng.integers(p, p + 8))
        kind = ["b3f", "uniform", "equal"][trial % 3]
        f, b, a = synth.random_tables(1700 + trial, n, kind)
        bw = synth.link_for(kind)
        plan = _plan(ap, f, b, a, bw)
        N = ap.ap_count(n, p)
        o = oracle_mod.Model(f, b, a, bw).exhaustive(p, m, 1, 2)
        ap.ap_search_heuristic(plan, p, m, 0x5EED, 2, 0, 64, 0, hk)
        torch.cuda.synchronize()
        th = int(hk.item()) >> 20
        for bound in (th, o["T"]):
            for mode in (0, 1, 2):
                ap.ap_search_exhaustive_bounded(plan, p, m, 1, 2, 0, N, mode, bound, out)
                torch.cuda.synchronize()
                res = ap.ap_decode(plan, 2, p, m, 1, 2, key=int(out[1].item()))
                assert int(out[0].item()) == o["T"]
                assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"]), (trial, mode)
        ap.ap_search_exhaustive_bounded(plan, p, m, 1, 2, 0, N, 2, o["T"] - 1, out)
        torch.cuda.synchronize()
        assert out.tolist() == [2**63 - 1, 2**63 - 1]
    with pytest.raises(ap.APError):
        ap.ap_search_exhaustive_bounded(plan, p, m, 1, 2, 0, N, 2, -1, out)


def test_eval_master_renormalised_beyond_u32(ap, oracle_mod):
    """ap_eval_batch on the u32 fast path renormalises its state instead of clamping it
    (Renorm, ap_master.cuh), T + master and T only: candidates whose T exceeds 2^32
    (C4's most unbalanced partitions at m = 100) are still exact, T and master equal to
    the oracle's."""
    import torch
    wl = synth.config(4)
    f, b, a = wl.arrays()
    plan = _plan(ap, f, b, a, wl.link_bytes_per_s)
    M = oracle_mod.Model.from_workload(wl)
    n, p, m = wl.n, wl.p, 100  # m = 100: the most unbalanced partitions pass 2^32 ns
    rows = [list(range(1, p)), list(range(n - p + 1, n)), [1, 2, 3, 4, 5, 6, 40],
            [20, 21, 22, 23, 24, 25, 26], [1, 30, 31, 32, 33, 34, 35]]
    rng = np.random.default_rng(5)
    while len(rows) < 64:
        rows.append(sorted(rng.choice(np.arange(1, n), p - 1, replace=False).tolist()))
    want = [M.simulate(p, m, r) for r in rows]
    assert sum(w["T"] >= 2 ** 32 for w in want) >= 3
    cuts = torch.tensor(rows, dtype=torch.int32, device="cuda")
    k1 = torch.ones(len(rows), dtype=torch.int32, device="cuda")
    T = torch.empty(len(rows), dtype=torch.int64, device="cuda")
    Ms = torch.empty(len(rows), dtype=torch.int32, device="cuda")
    ap.ap_eval_batch(plan, p, m, cuts, k1, T, Ms)
    torch.cuda.synchronize()
    assert T.tolist() == [w["T"] for w in want]
    assert Ms.tolist() == [w["master"] for w in want]
    # T only, k = 1..8: the offset-form sweep renormalises too (sim_fast_rn)
    ks = [1 + (i % 8) for i in range(len(rows))]
    wantk = [M.simulate(p, m, r, k=kk)["T"] for r, kk in zip(rows, ks)]
    assert sum(t >= 2 ** 32 for t in wantk) >= 3
    ap.ap_eval_batch(plan, p, m, cuts, torch.tensor(ks, dtype=torch.int32, device="cuda"), T)
    torch.cuda.synchronize()
    assert T.tolist() == wantk
