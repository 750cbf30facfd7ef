"""Critical-path and master parity at full size on the five configs (-m gpu).

North star: "bit-exact agreement with the CPU oracle on iteration time, argmin partition
and critical path".  For every config the partitions that matter are compared op by op
(stage, kind, micro-batch, piece, start, end) between ap_critical_path and the oracle's
explicit DAG backtrack (readings Q10/Q11), and T + master between
ap_eval_batch and the oracle, at EVERY k = 1..16:

* the oracle's own winners -- C1/C2 brute force, C3/C4 its exact LB-skipping
  enumeration, C5 the heuristic over all 65 536 restarts;
* the Algorithm 1 partition (the heuristic's start, T_ref);
* seeded random partitions.

The GPU's decoded winners (ap_decode: unrank + re-simulation + master from the device
critical path) are checked against the oracle's winners too, and the C5 winner's Slicer
sweep against the oracle's.  Every oracle input is the oracle's or synth's, never the
GPU's.
"""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu

K_ALL = 16


@pytest.fixture(scope="module")
def ap():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_cluster_liulldgl22_b200 as ap
    return ap


@pytest.fixture(scope="module")
def winners(oracle_mod):
    """Oracle argmins per config (computed on the host cores)."""
    out = {}
    for cfg in synth.ALL_CONFIGS:
        wl = synth.config(cfg)
        M = oracle_mod.Model.from_workload(wl)
        if cfg in (1, 2):
            o = M.exhaustive_parallel(wl.p, wl.m, wl.k_lo, wl.k_hi)
        elif cfg in (3, 4):
            o = M.exhaustive_bnb(wl.p, wl.m, wl.k_lo, wl.k_hi)
        else:
            o = M.heuristic_parallel(wl.p, wl.m, wl.seed, wl.radius, 0, wl.restarts)
        out[cfg] = (wl, M, o)
    return out


def _cases(wl, M, o):
    a1, _ = M.alg1(wl.p)
    rnd = synth.random_cuts(1000 + wl.n, wl.n, wl.p, 3)
    return [("winner", [int(x) for x in o["cuts"]]), ("alg1", [int(x) for x in a1])] + \
        [(f"random{i}", [int(x) for x in c]) for i, c in enumerate(rnd)]


@pytest.mark.parametrize("cfg", [1, 2, 3, 4, 5])
def test_critical_path_full_size_every_k(ap, winners, cfg):
    """ap_critical_path == oracle path op by op (times included), master and T, for the
    winner, the Algorithm 1 partition and random partitions, k = 1..16."""
    wl, M, o = winners[cfg]
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=0)
    n_ops = 0
    for name, cuts in _cases(wl, M, o):
        for k in range(1, K_ALL + 1):
            g = ap.ap_critical_path(plan, wl.p, wl.m, k, cuts)
            r = M.simulate(wl.p, wl.m, cuts, k=k, want_path=True)
            assert (g["T"], g["master"], g["path_len"]) == (r["T"], r["master"], r["path_len"]), \
                (cfg, name, k)
            assert g["path"] == r["path"], (cfg, name, k)
            n_ops += len(r["path"])
    assert n_ops > 5 * K_ALL * wl.p


@pytest.mark.parametrize("cfg", [1, 2, 3, 4, 5])
def test_eval_batch_master_full_size_every_k(ap, winners, cfg):
    """ap_eval_batch (T + master, the u32 bit-recording path where it applies and the
    exact fallback) == oracle on the same rows, every k = 1..16."""
    import torch
    wl, M, o = winners[cfg]
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=0)
    rows, ks = [], []
    for _, cuts in _cases(wl, M, o):
        for k in range(1, K_ALL + 1):
            rows.append(cuts); ks.append(k)
    c = torch.tensor(np.asarray(rows, np.int32), device="cuda")
    kk = torch.tensor(np.asarray(ks, np.int32), device="cuda")
    T = torch.empty(len(rows), dtype=torch.int64, device="cuda")
    Mv = torch.empty(len(rows), dtype=torch.int32, device="cuda")
    ap.ap_eval_batch(plan, wl.p, wl.m, c, kk, T, Mv)
    torch.cuda.synchronize()
    T, Mv = T.cpu().numpy(), Mv.cpu().numpy()
    for i, (cuts, k) in enumerate(zip(rows, ks)):
        r = M.simulate(wl.p, wl.m, cuts, k=k)
        assert (int(T[i]), int(Mv[i])) == (r["T"], r["master"]), (cfg, cuts, k)


@pytest.mark.parametrize("cfg", [1, 2, 3, 4])
def test_decoded_exhaustive_winner_master_and_path(ap, winners, cfg):
    """The GPU search (bench launch configuration) + ap_decode: the decoded winner's
    T, rank, k, cuts AND master equal the oracle's; its critical path at the winning k
    equals the oracle's op by op."""
    import torch
    wl, M, o = winners[cfg]
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=0)
    N = ap.ap_count(wl.n, wl.p)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    mode = ap.AP_SEARCH_FULL if cfg != 4 else ap.AP_SEARCH_PRUNED   # same key (tested)
    ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
    torch.cuda.synchronize()
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=int(key.item()))
    r = M.simulate(wl.p, wl.m, o["cuts"], k=o["k"], want_path=True)
    assert (res["time_ns"], res["rank"], res["k"], res["cuts"]) == \
        (o["T"], o["rank"], o["k"], [int(x) for x in o["cuts"]])
    assert res["master"] == r["master"]
    g = ap.ap_critical_path(plan, wl.p, wl.m, o["k"], [int(x) for x in o["cuts"]])
    assert g["path"] == r["path"]


def test_decoded_heuristic_winner_C5_slicer_and_paths(ap, winners):
    """C5: the 65 536-restart heuristic winner decoded on the GPU (cuts, T, master)
    equals the oracle's; its Slicer sweep k = 1..16 (T(k), best k) equals the oracle's,
    and so does the critical path at the Slicer's best k."""
    import torch
    wl, M, o = winners[5]
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=0)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, wl.restarts, 0, key)
    torch.cuda.synchronize()
    kv = int(key.item())
    assert (kv >> 20, kv & 0xFFFFF) == (o["T"], o["restart"])
    res = ap.ap_decode(plan, 1, wl.p, wl.m, seed=wl.seed, radius=wl.radius, key=kv)
    cuts = [int(x) for x in o["cuts"]]
    assert res["cuts"] == cuts and res["time_ns"] == o["T"]
    assert res["master"] == M.simulate(wl.p, wl.m, cuts)["master"]
    T, bk = ap.ap_slice_sweep(plan, wl.p, wl.m, cuts, wl.slice_k_max)
    oT, obk = M.slice_sweep(wl.p, wl.m, cuts, wl.slice_k_max)
    assert [int(x) for x in T] == [int(x) for x in oT] and bk == obk
    g = ap.ap_critical_path(plan, wl.p, wl.m, obk, cuts)
    r = M.simulate(wl.p, wl.m, cuts, k=obk, want_path=True)
    assert g["path"] == r["path"] and g["master"] == r["master"]
