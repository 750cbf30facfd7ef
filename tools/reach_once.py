"""C5 reachable-set search (65 536 restarts, vmax 1024) vs the greedy walk: time,
simulations, winner.  usage: reach_once.py [reps]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap
wl = synth.config(int(os.environ.get("CFG", "5")))
f, b, a = wl.arrays()
plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
key = torch.empty(1, dtype=torch.int64, device="cuda")
R = int(os.environ.get("R", "65536"))
for rep in range(int(sys.argv[1]) if len(sys.argv) > 1 else 3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    ap.ap_search_reachable(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 1024, key)
    kv = int(key.item()); t1 = time.perf_counter()
    kms, sims, tr = ap.ap_last_kernel_ms(), ap.ap_last_sims(), ap.ap_last_truncated()
    res = ap.ap_decode_reachable(plan, wl.p, wl.m, wl.seed, wl.radius, 1024, kv); t2 = time.perf_counter()
    print(f"reach  search {1e3*(t1-t0):.2f} ms (kernel {kms:.2f} ms, {sims} sims, {sims/kms*1e3:.3e} sims/s, {tr} truncated) decode {1e3*(t2-t1):.2f} ms T {res['time_ns']} r {res['restart']}", flush=True)
    torch.cuda.synchronize(); t0 = time.perf_counter()
    ap.ap_search_heuristic(plan, wl.p, wl.m, wl.seed, wl.radius, 0, R, 0, key)
    kv = int(key.item()); t1 = time.perf_counter()
    kms, sims = ap.ap_last_kernel_ms(), ap.ap_last_sims()
    print(f"greedy search {1e3*(t1-t0):.2f} ms (kernel {kms:.2f} ms, {sims} sims) T {kv >> 20} r {kv & 0xFFFFF}", flush=True)
