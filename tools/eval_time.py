"""ap_eval_batch device time (CUDA events, median of 7) on random valid partitions:
T only (k in [k_lo, k_hi]) and T + master (k = 1).  usage: eval_time.py CFG [log2 count]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 4
cnt = 1 << (int(sys.argv[2]) if len(sys.argv) > 2 else 22)
wl = synth.config(cfg)
f, b, a = wl.arrays()
plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
g = torch.Generator(device="cuda"); g.manual_seed(1234)
cuts = torch.sort(torch.argsort(torch.rand(cnt, wl.n - 1, device="cuda", generator=g), dim=1)
                  [:, : wl.p - 1] + 1, dim=1).values.to(torch.int32).contiguous()
ks = torch.randint(wl.k_lo, wl.k_hi + 1, (cnt,), device="cuda", generator=g, dtype=torch.int32)
k1 = torch.ones(cnt, dtype=torch.int32, device="cuda")
T = torch.empty(cnt, dtype=torch.int64, device="cuda")
M = torch.empty(cnt, dtype=torch.int32, device="cuda")
for name, kk, mm in (("T", ks, None), ("T+master(k=1)", k1, M)):
    ap.ap_eval_batch(plan, wl.p, wl.m, cuts, kk, T, mm)
    ts = []
    for _ in range(7):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); ap.ap_eval_batch(plan, wl.p, wl.m, cuts, kk, T, mm); e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ms = statistics.median(ts)
    print(f"{wl.name} eval {name}: {cnt} in {ms:.3f} ms = {cnt / ms * 1e3:.3e} sims/s", flush=True)
