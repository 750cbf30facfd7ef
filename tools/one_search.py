"""One search + decode + Slicer sweep of a config (for ncu launch lists).
usage: one_search.py CFG MODE"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_cluster_liulldgl22_b200 as ap
cfg = int(sys.argv[1]); mode = int(sys.argv[2])
wl = synth.config(cfg)
f, b, a = wl.arrays()
plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
N = ap.ap_count(wl.n, wl.p)
key = torch.empty(1, dtype=torch.int64, device="cuda")
for _ in range(2):
    ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=int(key.item()))
    ap.ap_slice_sweep(plan, wl.p, wl.m, res["cuts"], wl.k_hi)
torch.cuda.synchronize()
print(res)
