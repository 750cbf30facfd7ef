"""Time the three exhaustive search modes (same key) on C2-C4 (diagnostic)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap
for cfg in [int(a) for a in sys.argv[1:]] or [2, 3, 4]:
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    key = torch.empty(1, dtype=torch.int64, device="cuda")
    for mode in (0, 1, 2):
        for rep in range(3):
            torch.cuda.synchronize(); t0 = time.perf_counter()
            ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
            kv = int(key.item()); dt = time.perf_counter() - t0
        print(wl.name, "mode", mode, f"{dt*1e3:.2f} ms", f"kernel {ap.ap_last_kernel_ms():.2f} ms",
              f"{N*(wl.k_hi-wl.k_lo+1)/dt:.3e} candidates/s", kv, flush=True)
