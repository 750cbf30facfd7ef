"""Host-side cost of one search call (launches only, no sync) vs its device time:
C3 pruned and C5 heuristic.  usage: host_overhead.py"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_cluster_liulldgl22_b200 as ap

for cfg, mode in ((3, 2), (4, 2)):
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    for _ in range(5):
        ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
    torch.cuda.synchronize()
    reps = 50
    t0 = time.perf_counter()
    for _ in range(reps):
        ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    print(f"{wl.name} mode {mode}: host {1e6*(t1-t0)/reps:.1f} us/call, wall {1e6*(t2-t0)/reps:.1f} us/call "
          f"(back to back, stream-ordered), kernel {1e3*ap.ap_last_kernel_ms():.1f} us", flush=True)
    kv = int(key.item())
    t0 = time.perf_counter()
    for _ in range(20):
        res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=kv)
    t1 = time.perf_counter()
    for _ in range(20):
        ap.ap_slice_sweep(plan, wl.p, wl.m, res["cuts"], wl.k_hi)
    t2 = time.perf_counter()
    print(f"   decode {1e6*(t1-t0)/20:.1f} us, slice sweep {1e6*(t2-t1)/20:.1f} us", flush=True)
