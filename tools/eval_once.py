"""ap_eval_batch throughput on C4 (random valid partitions, k in 1..8): T only and T +
master.  usage: eval_once.py [count_log2]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap

wl = synth.config(int(os.environ.get("AP_CFG", "4")))
f, b, a = wl.arrays()
plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
cnt = 1 << (int(sys.argv[1]) if len(sys.argv) > 1 else 22)
rng = np.random.default_rng(5)
cuts = np.sort(np.argsort(rng.random((cnt, wl.n - 1)), axis=1)[:, : wl.p - 1] + 1, axis=1).astype(np.int32)
ks = rng.integers(wl.k_lo, wl.k_hi + 1, cnt).astype(np.int32)
d_cuts = torch.from_numpy(cuts).cuda()
d_k = torch.from_numpy(ks).cuda()
d_k1 = torch.ones(cnt, dtype=torch.int32, device="cuda")
T = torch.empty(cnt, dtype=torch.int64, device="cuda")
Mst = torch.empty(cnt, dtype=torch.int32, device="cuda")
for name, kk, mm in (("T only, k 1..K", d_k, None), ("T + master, k = 1", d_k1, Mst)):
    for rep in range(3):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        ap.ap_eval_batch(plan, wl.p, wl.m, d_cuts, kk, T, mm)
        torch.cuda.synchronize(); dt = time.perf_counter() - t0
    print(f"{wl.name} eval {name}: {cnt} candidates {1e3*dt:.2f} ms {cnt/dt:.3e} sims/s "
          f"T[0..3] {T[:3].tolist()} min T {int(T.min())}", flush=True)
