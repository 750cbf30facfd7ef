"""Heuristic quality vs the exact optimum (NEXT N1): C2-C4 exhaustive k=1 optimum,
the greedy walk (adjust_mode 0), the Eq. (1) mode (adjust_mode 1) and the
reachable-set search, each with 1 / 256 / 65 536 restarts; C5 against the certified
minLB.  Prints a markdown table.  All on the GPU through the C ABI."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap
from paper_conf_cluster_liulldgl22_b200.search import search_exhaustive

key = torch.empty(1, dtype=torch.int64, device="cuda")
rows = []
print("| config | reference T (ns) | restarts | greedy | eq1 | reachable | reachable sims |")
print("|---|---|---|---|---|---|---|")
for cfg in (2, 3, 4, 5):
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    if cfg < 5:
        ref = search_exhaustive(plan, wl.p, wl.m, 1, 1)["time_ns"]
        label = f"{ref} (exhaustive, k=1)"
    else:
        ref, _ = ap.ap_min_lower_bound(plan, wl.p, wl.m, 1)
        label = f"{ref} (certified minLB)"
    for R in (1, 256, 65536):
        out = []
        for kind in ("greedy", "eq1", "reach"):
            if kind == "reach":
                ap.ap_search_reachable(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 1024, key)
            else:
                ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R,
                                       1 if kind == "eq1" else 0, key)
            T = int(key.item()) >> 20
            out.append(f"{T} (+{100.0 * (T - ref) / ref:.2f}%)")
        sims = ap.ap_last_sims()
        print(f"| C{cfg} | {label} | {R} | {out[0]} | {out[1]} | {out[2]} | {sims} |", flush=True)
