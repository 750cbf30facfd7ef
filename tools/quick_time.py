"""Quick timing probe of the exhaustive sweep (not the bench; see bench.py)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap

for cfg in [int(a) for a in sys.argv[1:]] or [3, 4]:
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    for rep in range(3):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        ap.ap_search_exhaustive(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, key)
        torch.cuda.synchronize(); dt = time.perf_counter() - t0
    info = ap.ap_last_launch()
    sims = N * (wl.k_hi - wl.k_lo + 1)
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=int(key.item()))
    print(wl.name, f"{dt*1e3:.1f} ms", f"{sims/dt:.3e} sims/s", info, res, flush=True)
