"""Small run of every kernel family, for compute-sanitizer (C1/C2 sizes)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap
for cfg in (1, 2):
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    for mode in (0, 1, 2):
        ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
    torch.cuda.synchronize()
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=int(key.item()))
    ap.ap_critical_path(plan, wl.p, wl.m, 2, res["cuts"])
    ap.ap_slice_sweep(plan, wl.p, wl.m, res["cuts"], 8)
    ap.ap_slice_sweep_paper(plan, wl.p, wl.m, res["cuts"], 2, wl.p)
    ap.ap_slicer_alg2(plan, wl.p, res["cuts"], 1)
    ap.ap_alg1(plan, wl.p)
    for am in (0, 1):
        ap.ap_search_heuristic(plan, wl.p, wl.m, 0x5EED, 2, 0, 64, am, key)
        torch.cuda.synchronize()
        ap.ap_decode(plan, 1, wl.p, wl.m, seed=0x5EED, radius=2, adjust_mode=am, key=int(key.item()))
    cuts = torch.tensor(synth.random_cuts(1, wl.n, wl.p, 64), device="cuda")
    ks = torch.randint(1, 5, (64,), dtype=torch.int32, device="cuda")
    T = torch.empty(64, dtype=torch.int64, device="cuda"); M = torch.empty(64, dtype=torch.int32, device="cuda")
    ap.ap_eval_batch(plan, wl.p, wl.m, cuts, ks, T, M)
    torch.cuda.synchronize()
print("sanitize run ok")
