"""C3/C4: pruned search bounded by the heuristic's attained plan (diagnostic, not the bench).
Times (a) PRUNED alone, (b) PRUNED bounded at the known optimum (ideal bound), (c) heuristic
with R restarts + slice sweep of its winner + PRUNED bounded by that T; keys must agree."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_liulldgl22_b200 as ap


def best(fn, reps=5):
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        r = fn(); torch.cuda.synchronize(); ts.append(time.perf_counter() - t0)
    return r, min(ts) * 1e3


for cfg in [int(a) for a in sys.argv[1:]] or [3, 4]:
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s)
    N = ap.ap_count(wl.n, wl.p)
    out = torch.empty(2, dtype=torch.int64, device="cuda")
    hk = torch.empty(1, dtype=torch.int64, device="cuda")
    PR = ap.AP_SEARCH_PRUNED

    def plain():
        ap.ap_search_exhaustive2(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, PR, out)
        return (int(out[0]), int(out[1]))
    ref, t_plain = best(plain)

    def ideal():
        ap.ap_search_exhaustive_bounded(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, PR, ref[0], out)
        return (int(out[0]), int(out[1]))
    r_ideal, t_ideal = best(ideal)
    print(wl.name, f"plain {t_plain:.3f} ms  ideal-bound {t_ideal:.3f} ms", ref == r_ideal, flush=True)
    for R in (1, 64, 1024):
        def heur():
            ap.ap_search_heuristic(plan, wl.p, wl.m, 1, 2, 0, R, 0, hk)
            h = ap.ap_decode(plan, 1, wl.p, wl.m, seed=1, radius=2, key=int(hk.item()))
            T, _ = ap.ap_slice_sweep(plan, wl.p, wl.m, h["cuts"], wl.k_hi)
            tb = int(T[wl.k_lo - 1:wl.k_hi].min())
            ap.ap_search_exhaustive_bounded(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, PR, tb, out)
            return (int(out[0]), int(out[1])), tb
        (r, tb), t = best(heur)
        print(f"  heur R={R}: bound {tb} (opt {ref[0]}) total {t:.3f} ms same={r == ref}", flush=True)
