"""The exhaustive search is stream-ordered end to end (include/ap.h): nothing inside it
waits for the device, so it can be captured in a CUDA graph and replayed (-m gpu).

C3 in the pruned mode and C2 in the full mode (k = 1..4) are captured once with
torch.cuda.graph and replayed; the replayed key equals the eagerly computed one and
decodes to the oracle's argmin.  Round 1 read T_ref on the host inside every search,
which made this impossible.
"""
import pytest

import synth

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("cfg,mode", [(3, 2), (2, 0)])
def test_search_captured_in_cuda_graph(oracle_mod, cfg, mode):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_cluster_liulldgl22_b200 as ap
    wl = synth.config(cfg)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=0)
    N = ap.ap_count(wl.n, wl.p)
    eager = torch.empty(1, dtype=torch.int64, device="cuda")
    ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, eager)
    torch.cuda.synchronize()
    key = torch.full((1,), -7, dtype=torch.int64, device="cuda")
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):  # warm-up on a side stream, as torch recommends
        ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, 0, N, mode, key)
    key.fill_(-7)
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    assert int(key.item()) == int(eager.item())
    res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=int(key.item()))
    M = oracle_mod.Model.from_workload(wl)
    o = (M.exhaustive_parallel(wl.p, wl.m, wl.k_lo, wl.k_hi) if cfg == 2
         else M.exhaustive_bnb(wl.p, wl.m, wl.k_lo, wl.k_hi))
    assert (res["time_ns"], res["rank"], res["k"]) == (o["T"], o["rank"], o["k"])
