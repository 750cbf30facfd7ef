"""Probe: pruned exact search (mode 2, two-phase key) over sampled C5 rank windows, to
estimate the cost of an exact C5 optimum.  usage: c5_pruned_probe.py [span] [windows]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch, synth
import paper_conf_cluster_liulldgl22_b200 as ap
wl = synth.config(5)
f, b, a = wl.arrays()
plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
N = ap.ap_count(wl.n, wl.p)
span = int(float(sys.argv[1])) if len(sys.argv) > 1 else 10**14
W = int(sys.argv[2]) if len(sys.argv) > 2 else 16
out = torch.empty(2, dtype=torch.int64, device="cuda")
rng = np.random.default_rng(3)
ap.ap_search_exhaustive2(plan, wl.p, wl.m, 1, 1, 0, 10**6, 2, out)
tot = 0.0
found = []
for w in range(W):
    lo = int(rng.integers(0, N - span))
    torch.cuda.synchronize(); t0 = time.perf_counter()
    ap.ap_search_exhaustive2(plan, wl.p, wl.m, 1, 1, lo, lo + span, 2, out)
    torch.cuda.synchronize(); dt = time.perf_counter() - t0
    tot += dt
    o = out.tolist()
    if o[0] != 2**63 - 1:
        found.append(o)
    print(f"window {w} lo {lo} {dt*1e3:.1f} ms {o}", flush=True)
    if dt > 30:
        break
mean = tot / (w + 1)
print(f"mean {mean*1e3:.1f} ms per {span:.0e} ranks -> full space ~{mean * N / span:.0f} s on one GPU; found {found}")
