"""Debug probe: T + master through ap_eval_batch (fast kernel) on a few configs vs oracle."""
import os, sys, faulthandler
faulthandler.enable()
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth, oracle
import paper_conf_cluster_liulldgl22_b200 as ap
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 1
cnt = int(sys.argv[2]) if len(sys.argv) > 2 else 8
wl = synth.config(cfg)
f, b, a = wl.arrays()
plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
M = oracle.Model.from_workload(wl)
cuts = synth.random_cuts(3, wl.n, wl.p, cnt)
c = torch.tensor(np.asarray(cuts, np.int32), device="cuda")
k = torch.ones(cnt, dtype=torch.int32, device="cuda")
T = torch.empty(cnt, dtype=torch.int64, device="cuda"); Mv = torch.empty(cnt, dtype=torch.int32, device="cuda")
print("launch", flush=True)
ap.ap_eval_batch(plan, wl.p, wl.m, c, k, T, Mv)
print("sync", flush=True)
torch.cuda.synchronize()
bad = 0
for i in range(cnt):
    r = M.simulate(wl.p, wl.m, cuts[i])
    if (int(T[i]), int(Mv[i])) != (r["T"], r["master"]):
        bad += 1
        if bad < 5: print("MISMATCH", i, list(cuts[i]), int(T[i]), int(Mv[i]), r["T"], r["master"])
print("cfg", cfg, "bad", bad, "of", cnt, flush=True)
