"""Small run of every kernel family, for compute-sanitizer (C1/C2 sizes plus small
synthetic tables for the p = 16 / saturating / memory / two-phase paths).

Entry points of include/ap.h driven here: ap_plan_create/destroy, ap_plan_set_memory,
ap_count, ap_eval_batch (T only and T + master: k_eval_fast and the generic k_eval),
ap_search_exhaustive(_mode) in all three modes (k_alg1, k_eval*, k_sweep_prep,
k_sweep_exact u32 + int64, k_sweep_generic), AP_SEARCH_MEMORY, ap_search_exhaustive2 and
ap_search_exhaustive_bounded in all three modes (k_reduce2), ap_key2_select, the
key-packing overflow (AP_KEY_RANGE), ap_search_heuristic in both adjust modes (the warp
pool k_heur_pool, the lane kernel k_heur, its exact redo pass), ap_search_reachable with
vmax <= 2048 (k_reach_pool) and > 2048 (k_reach), ap_decode modes 0/1/2,
ap_decode_reachable, ap_slice_sweep, ap_slice_sweep_paper, ap_slicer_alg2,
ap_critical_path (k_cpath), ap_alg1, ap_min_lower_bound (k_minlb)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap


def dev(x, dt=torch.int32):
    return torch.tensor(np.asarray(x), dtype=dt, device="cuda")


key = torch.empty(1, dtype=torch.int64, device="cuda")
two = torch.empty(2, dtype=torch.int64, device="cuda")
for cfg in (1, 2):
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    for mode in (0, 1, 2):
        ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
        ap.ap_search_exhaustive2(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, two)
        ap.ap_search_exhaustive_bounded(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode,
                                        1 << 40, two)
    torch.cuda.synchronize()
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=int(key.item()))
    idx = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_key2_select(two, two[:1].clone(), idx)
    torch.cuda.synchronize()
    ap.ap_decode(plan, 2, wl.p, wl.m, wl.k_lo, wl.k_hi, key=int(idx.item()))
    ap.ap_critical_path(plan, wl.p, wl.m, 2, res["cuts"])
    ap.ap_slice_sweep(plan, wl.p, wl.m, res["cuts"], 8)
    ap.ap_slice_sweep_paper(plan, wl.p, wl.m, res["cuts"], 2, wl.p)
    ap.ap_slicer_alg2(plan, wl.p, res["cuts"], 1)
    ap.ap_alg1(plan, wl.p)
    ap.ap_min_lower_bound(plan, wl.p, wl.m, 4)
    for am in (0, 1):
        ap.ap_search_heuristic(plan, wl.p, wl.m, 0x5EED, 2, 0, 64, am, key)
        torch.cuda.synchronize()
        ap.ap_decode(plan, 1, wl.p, wl.m, seed=0x5EED, radius=2, adjust_mode=am, key=int(key.item()))
    for vmax in (64, 4096):  # k_reach_pool (vmax <= 2048) and k_reach
        ap.ap_search_reachable(plan, wl.p, wl.m, 0x5EED, 2, 0, 32, vmax, key)
        torch.cuda.synchronize()
        ap.ap_decode_reachable(plan, wl.p, wl.m, 0x5EED, 2, vmax, int(key.item()))
    cuts = dev(synth.random_cuts(1, wl.n, wl.p, 64))
    ks = torch.randint(1, 5, (64,), dtype=torch.int32, device="cuda")
    T = torch.empty(64, dtype=torch.int64, device="cuda"); M = torch.empty(64, dtype=torch.int32, device="cuda")
    ap.ap_eval_batch(plan, wl.p, wl.m, cuts, ks, T, M)
    ap.ap_eval_batch(plan, wl.p, wl.m, cuts, ks, T, None)
    # memory mode (N4): a cap that admits part of the space
    ap.ap_plan_set_memory(plan, np.full(wl.n, 1 << 20, np.int64), np.full(wl.n, 1 << 18, np.int64),
                          (wl.n // 2) << 20)
    ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, 1, 1, 0, N, ap.AP_SEARCH_MEMORY, key)
    ap.ap_search_exhaustive2(plan, wl.p, wl.m, 1, 1, 0, N, ap.AP_SEARCH_MEMORY, two)
    torch.cuda.synchronize()
    plan.close()

# p = 16 (the C5 kernels' template) on a small model, heuristic + T + master eval
f, b, a = synth.random_tables(3, 24, "b3f")
plan = ap.ap_plan_create(f, b, a, synth.LINK_BYTES_PER_S)
ap.ap_search_heuristic(plan, 16, 20, 0x5EED, 2, 0, 48, 0, key)
cuts = dev(synth.random_cuts(2, 24, 16, 32))
T = torch.empty(32, dtype=torch.int64, device="cuda"); M = torch.empty(32, dtype=torch.int32, device="cuda")
ap.ap_eval_batch(plan, 16, 20, cuts, None, T, M)
torch.cuda.synchronize()
# saturating fast paths: every u32 simulation saturates -> exact redo passes
os.environ["AP_HEUR_S"] = "1000"
os.environ["AP_EVAL_S"] = "1000"
ap.ap_search_heuristic(plan, 16, 20, 0x5EED, 2, 0, 16, 0, key)
ap.ap_eval_batch(plan, 16, 20, cuts, None, T, M)
torch.cuda.synchronize()
del os.environ["AP_HEUR_S"], os.environ["AP_EVAL_S"]
plan.close()

# key-packing overflow: the device writes AP_KEY_RANGE and no sweep runs
f, b, a = synth.random_tables(40, 30, "uniform", fmax=1 << 44)
plan = ap.ap_plan_create(f, b, a, synth.link_for("uniform"))
ap.ap_search_exhaustive(plan, 4, 16, 1, 4, 0, ap.ap_count(30, 4), key)
torch.cuda.synchronize()
assert int(key.item()) == ap.AP_KEY_RANGE
plan.close()
print("sanitize run ok")
