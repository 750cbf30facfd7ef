"""Exact C5 optimum (k = 1) by the pruned exhaustive search bounded by the heuristic's
result (ap_search_exhaustive_bounded, mode PRUNED), over the whole 1.5e17-partition
space in W windows.  usage: c5_exact.py [windows] [budget_s] [probe]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch, synth
import paper_conf_cluster_liulldgl22_b200 as ap
W = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
budget = float(sys.argv[2]) if len(sys.argv) > 2 else 600.0
probe = len(sys.argv) > 3 and sys.argv[3] == "probe"
wl = synth.config(5)
f, b, a = wl.arrays()
plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
N = ap.ap_count(wl.n, wl.p)
hk = torch.empty(1, dtype=torch.int64, device="cuda")
ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, wl.restarts, 0, hk)
th = int(hk.item()) >> 20
print(f"N {N}; heuristic T {th}; bound = {th}", flush=True)
out = torch.empty(2, dtype=torch.int64, device="cuda")
edges = [N * i // W for i in range(W + 1)]
order = range(W)
if probe:
    order = np.random.default_rng(7).permutation(W)[: max(1, W // 32)]
best = (2**63 - 1, 2**63 - 1)
t_start = time.perf_counter()
done = 0
for w in order:
    lo, hi = edges[w], edges[w + 1]
    torch.cuda.synchronize(); t0 = time.perf_counter()
    ap.ap_search_exhaustive_bounded(plan, wl.p, wl.m, 1, 1, lo, hi, 2, th, out)
    torch.cuda.synchronize(); dt = time.perf_counter() - t0
    o = tuple(out.tolist())
    best = min(best, o)
    done += 1
    if dt > 1.0 or o[0] != 2**63 - 1:
        print(f"window {w}/{W}: {dt:.2f} s {o}", flush=True)
    if time.perf_counter() - t_start > budget:
        break
el = time.perf_counter() - t_start
print(f"{done} of {W} windows in {el:.1f} s -> full space ~{el * W / done:.0f} s on one GPU", flush=True)
if not probe and done == W:
    res = ap.ap_decode(plan, 2, wl.p, wl.m, 1, 1, key=best[1])
    print(f"EXACT C5 optimum T* {res['time_ns']} cuts {res['cuts']} master {res['master']} "
          f"(heuristic {th}, gap {(th - res['time_ns']) / res['time_ns']:.4%}) in {el:.1f} s", flush=True)
