"""Host-side per-call time breakdown of one bench step (diagnostic)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 4
wl = synth.config(cfg)
f, b, a = wl.arrays()
plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
N = ap.ap_count(wl.n, wl.p)
key = torch.empty(1, dtype=torch.int64, device="cuda")
for rep in range(4):
    t = {}
    torch.cuda.synchronize()
    t0 = time.perf_counter(); pl2 = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s); t["plan_create"] = time.perf_counter() - t0
    t0 = time.perf_counter(); pl2.close(); t["plan_destroy"] = time.perf_counter() - t0
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ap.ap_search_exhaustive(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, key)
    t["search_call"] = time.perf_counter() - t0
    torch.cuda.synchronize()
    t["search_done"] = time.perf_counter() - t0
    t["kernel"] = ap.ap_last_kernel_ms() / 1e3
    t1 = time.perf_counter(); kv = int(key.item()); t["item"] = time.perf_counter() - t1
    t1 = time.perf_counter(); res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=kv); t["decode"] = time.perf_counter() - t1
    t1 = time.perf_counter(); ap.ap_slice_sweep(plan, wl.p, wl.m, res["cuts"], wl.k_hi); t["slice"] = time.perf_counter() - t1
    t1 = time.perf_counter(); ap.ap_alg1(plan, wl.p); t["alg1_call"] = time.perf_counter() - t1
    print({k: round(v * 1e3, 3) for k, v in t.items()}, flush=True)

# e2e-style loop: create -> search -> decode -> destroy
for rep in range(4):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    pl = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    t1 = time.perf_counter()
    ap.ap_search_exhaustive(pl, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, key)
    t2 = time.perf_counter()
    kv = int(key.item()); t3 = time.perf_counter()
    res = ap.ap_decode(pl, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=kv); t4 = time.perf_counter()
    pl.close(); t5 = time.perf_counter()
    print({"create": round((t1-t0)*1e3,3), "search_call": round((t2-t1)*1e3,3), "item": round((t3-t2)*1e3,3), "decode": round((t4-t3)*1e3,3), "destroy": round((t5-t4)*1e3,3), "kernel": round(ap.ap_last_kernel_ms(),3)}, flush=True)
