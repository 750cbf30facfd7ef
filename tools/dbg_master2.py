import os, sys, atexit, traceback
atexit.register(lambda: print("atexit reached", flush=True))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
try:
    import numpy as np, torch, synth
    import paper_conf_cluster_liulldgl22_b200 as ap
    wl = synth.config(1)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    cuts = synth.random_cuts(3, wl.n, wl.p, 4)
    c = torch.tensor(np.asarray(cuts, np.int32), device="cuda")
    T = torch.empty(4, dtype=torch.int64, device="cuda"); Mv = torch.empty(4, dtype=torch.int32, device="cuda")
    print("T only", flush=True)
    ap.ap_eval_batch(plan, wl.p, wl.m, c, None, T, None); torch.cuda.synchronize()
    print("T only ok", T.tolist(), flush=True)
    ap.ap_eval_batch(plan, wl.p, wl.m, c, None, T, Mv)
    print("returned", flush=True)
    torch.cuda.synchronize()
    print("ok", T.tolist(), Mv.tolist(), flush=True)
except BaseException as e:
    print("EXC", repr(e), flush=True)
    traceback.print_exc()
