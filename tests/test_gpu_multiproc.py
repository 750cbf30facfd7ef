"""The sharded search through a REAL process group with device keys (-m gpu).

Two ranks (torch.multiprocessing spawn, backend gloo) share cuda:0 -- a one-GPU box
cannot host two NCCL ranks on one device.  Every rank runs the public orchestration
layer (search.search_exhaustive / search.search_heuristic): its contiguous shard on the
GPU, then all_reduce(MIN) of the kernel-written int64 key (device tensor), then an
independent decode.  Covered: C2 (k = 1..4), C3, the
two-phase reduction (forced, plus the automatic fallback on tables whose packed key
does not fit), a shard layout with an empty rank, and the C5 heuristic over 4 096
restarts.  The parent compares every rank's result with the oracle.
"""
import os
import socket

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _big_tables():
    """Tables whose optimum needs ~51 bits, so T << rb | index does not fit in 63 bits
    and the search must take the two-phase reduction."""
    f, b, a = synth.random_tables(21, 14, "uniform")
    return f * (1 << 30), b * (1 << 30), a


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import paper_conf_cluster_liulldgl22_b200 as ap
        from paper_conf_cluster_liulldgl22_b200 import search
        out = {}
        for cfg in (2, 3):
            wl = synth.config(cfg)
            f, b, a = wl.arrays()
            plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=0)
            r = search.search_exhaustive(plan, wl.p, wl.m, wl.k_lo, wl.k_hi)
            out[f"C{cfg}"] = (r["time_ns"], r["rank"], r["k"], r["cuts"], r["master"],
                              r["shard"], r["two_phase"])
            if cfg == 2:
                r = search.search_exhaustive(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, two_phase=True)
                out["C2_two_phase"] = (r["time_ns"], r["rank"], r["k"], r["cuts"], r["two_phase"])
        f, b, a = _big_tables()
        plan = ap.ap_plan_create(f, b, a, 10**9, device=0)
        r = search.search_exhaustive(plan, 5, 9, 1, 3)
        out["big"] = (r["time_ns"], r["rank"], r["k"], r["two_phase"])
        # 3 stages on 3 blocks: N = 1 < world, so rank 0's shard is empty
        f3, b3, a3 = synth.random_tables(4, 3, "uniform")
        plan = ap.ap_plan_create(f3, b3, a3, synth.LINK_BYTES_PER_S, device=0)
        r = search.search_exhaustive(plan, 3, 4, 1, 2)
        out["tiny"] = (r["time_ns"], r["rank"], r["k"], r["shard"])
        # the same with costs whose packed key does not fit: every rank must still take
        # the same (two-phase) branch although rank 0 has nothing to search
        plan = ap.ap_plan_create(f3 * (1 << 37), b3 * (1 << 37), a3, synth.LINK_BYTES_PER_S,
                                 device=0)
        r = search.search_exhaustive(plan, 3, 4, 1, 16)
        out["tinybig"] = (r["time_ns"], r["rank"], r["k"], r["two_phase"], r["shard"])
        wl = synth.config(5)
        f, b, a = wl.arrays()
        plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=0)
        h = search.search_heuristic(plan, wl.p, wl.m, 4096, wl.seed, wl.radius)
        out["C5"] = (h["time_ns"], h["restart"], h["cuts"], h["shard"])
        q.put((rank, out))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, repr(e) + "\n" + traceback.format_exc()))


def test_two_ranks_on_one_gpu_real_process_group(oracle_mod):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert isinstance(res[r], dict), res[r]
    # shards differ, everything else is identical on both ranks
    for name, si in (("C2", 5), ("C3", 5), ("tiny", 3), ("C5", 3)):
        a0 = res[0][name][:si] + res[0][name][si + 1:]
        a1 = res[1][name][:si] + res[1][name][si + 1:]
        assert a0 == a1, name
        assert res[0][name][si] != res[1][name][si], name
    assert res[0]["C2_two_phase"] == res[1]["C2_two_phase"]
    assert res[0]["big"] == res[1]["big"]
    for cfg in (2, 3):
        wl = synth.config(cfg)
        M = oracle_mod.Model.from_workload(wl)
        o = (M.exhaustive_parallel(wl.p, wl.m, wl.k_lo, wl.k_hi) if cfg == 2
             else M.exhaustive_bnb(wl.p, wl.m, wl.k_lo, wl.k_hi))
        T, rk, k, cuts, master, _, two = res[0][f"C{cfg}"]
        assert (T, rk, k, cuts) == (o["T"], o["rank"], o["k"], [int(x) for x in o["cuts"]])
        assert master == M.simulate(wl.p, wl.m, o["cuts"], k=o["k"])["master"]
        assert not two
        if cfg == 2:
            assert res[0]["C2_two_phase"] == (o["T"], o["rank"], o["k"],
                                             [int(x) for x in o["cuts"]], True)
    f, b, a = _big_tables()
    o = oracle_mod.Model(f, b, a, 10**9).exhaustive(5, 9, 1, 3)
    assert res[0]["big"] == (o["T"], o["rank"], o["k"], True)
    f3, b3, a3 = synth.random_tables(4, 3, "uniform")
    o = oracle_mod.Model(f3, b3, a3, synth.LINK_BYTES_PER_S).exhaustive(3, 4, 1, 2)
    assert res[0]["tiny"][:3] == (o["T"], o["rank"], o["k"])
    assert {res[0]["tiny"][3], res[1]["tiny"][3]} == {(0, 0), (0, 1)}
    o = oracle_mod.Model(f3 * (1 << 37), b3 * (1 << 37), a3,
                         synth.LINK_BYTES_PER_S).exhaustive(3, 4, 1, 16)
    assert res[0]["tinybig"][:4] == (o["T"], o["rank"], o["k"], True)
    assert res[0]["tinybig"][:4] == res[1]["tinybig"][:4]
    wl = synth.config(5)
    o = oracle_mod.Model.from_workload(wl).heuristic_parallel(wl.p, wl.m, wl.seed, wl.radius, 0, 4096)
    assert res[0]["C5"][:3] == (o["T"], o["restart"], [int(x) for x in o["cuts"]])
