"""Multi-process host logic on CPU (gloo, world size 2): contiguous shards, ONE
all_reduce(MIN) of the packed int64 key, independent decode on every rank
(DESIGN.md §6).  Per-rank keys come from the oracle on that rank's shard, packed
in the layout the C ABI documents; the reduced key must decode to the global
oracle argmin."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _two_phase_cases():
    import numpy as np
    import synth
    cases = {}
    f, b, a = synth.random_tables(5, 12, "equal")
    cases["equal"] = (f, b, a, synth.link_for("equal"), 3, 4, 1, 2)
    f, b, a = synth.random_tables(6, 14, "small")
    cases["small"] = (f, b, a, synth.link_for("small"), 4, 5, 1, 3)
    f, b, a = synth.random_tables(7, 9, "uniform")
    cases["tiny"] = (f, b, a, synth.link_for("uniform"), 9, 2, 1, 1)  # N = 1: one rank empty
    return cases


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import oracle
        import synth
        from paper_conf_cluster_liulldgl22_b200.search import (
            INT64_MAX, min_allreduce_key, pack_exhaustive_key, shard, unpack_exhaustive_key,
            unpack_heuristic_key)
        out = {}
        for cfg in (1, 2):
            wl = synth.config(cfg)
            M = oracle.Model.from_workload(wl)
            N = oracle.count(wl.n, wl.p)
            lo, hi = shard(N, rank, world)
            r = M.exhaustive(wl.p, wl.m, wl.k_lo, wl.k_hi, lo, hi)
            key = torch.tensor([pack_exhaustive_key(r["T"], r["rank"], r["k"], N, wl.k_lo, wl.k_hi)
                                if r["sims"] else INT64_MAX], dtype=torch.int64)
            min_allreduce_key(key, dist)
            out[cfg] = unpack_exhaustive_key(int(key.item()), N, wl.k_lo, wl.k_hi)
        wl = synth.config(2)
        M = oracle.Model.from_workload(wl)
        lo, hi = shard(256, rank, world)
        h = M.heuristic(wl.p, wl.m, wl.seed, wl.radius, lo, hi)
        key = torch.tensor([(h["T"] << 20) | h["restart"]], dtype=torch.int64)
        min_allreduce_key(key, dist)
        out["heur"] = unpack_heuristic_key(int(key.item()))
        # two-phase reduction (NEXT N3): per-rank (T, index), T* first, then the least
        # index among the ranks holding T*.  'equal' tables tie across the shards.
        from paper_conf_cluster_liulldgl22_b200.search import two_phase_reduce

        def cpu_select(loc, ts, idx):
            hit = int(loc[0]) == int(ts[0]) and int(loc[0]) != INT64_MAX
            idx.fill_(int(loc[1]) if hit else INT64_MAX)

        tp = {}
        for name, (f, b, a, bw, p, m, k_lo, k_hi) in _two_phase_cases().items():
            M = oracle.Model(f, b, a, bw)
            N = oracle.count(len(f), p)
            K = k_hi - k_lo + 1
            lo, hi = shard(N, rank, world)
            r = M.exhaustive(p, m, k_lo, k_hi, lo, hi) if hi > lo else {"sims": 0}
            loc = torch.tensor([r["T"], r["rank"] * K + r["k"] - k_lo] if r["sims"]
                               else [INT64_MAX, INT64_MAX], dtype=torch.int64)
            T, idx = two_phase_reduce(loc, dist, None, cpu_select)
            tp[name] = (T, idx // K, k_lo + idx % K)
        out["two_phase"] = tp
        q.put((rank, out))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))


def test_two_rank_gloo_shard_reduce_decode(oracle_mod):
    import synth
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert isinstance(res[r], dict), res[r]
    assert res[0] == res[1]
    for cfg in (1, 2):
        wl = synth.config(cfg)
        o = oracle_mod.Model.from_workload(wl).exhaustive(wl.p, wl.m, wl.k_lo, wl.k_hi)
        assert res[0][cfg] == (o["T"], o["rank"], o["k"])
    wl = synth.config(2)
    o = oracle_mod.Model.from_workload(wl).heuristic(wl.p, wl.m, wl.seed, wl.radius, 0, 256)
    assert res[0]["heur"] == (o["T"], o["restart"])
    for name, (f, b, a, bw, p, m, k_lo, k_hi) in _two_phase_cases().items():
        o = oracle_mod.Model(f, b, a, bw).exhaustive(p, m, k_lo, k_hi)
        assert res[0]["two_phase"][name] == (o["T"], o["rank"], o["k"]), name


def test_shard_covers_exactly():
    from paper_conf_cluster_liulldgl22_b200.search import shard
    for total in (0, 1, 7, 84, 18424, 696190560):
        for world in (1, 2, 3, 8, 13):
            edges = [shard(total, r, world) for r in range(world)]
            assert edges[0][0] == 0 and edges[-1][1] == total
            for (a, b), (c, d) in zip(edges, edges[1:]):
                assert b == c and a <= b
            sizes = [b - a for a, b in edges]
            assert max(sizes) - min(sizes) <= 1


def test_key_order_is_lexicographic():
    """Packed keys order exactly as (T, rank, k): MIN over keys == lex min."""
    import random
    from paper_conf_cluster_liulldgl22_b200.search import pack_exhaustive_key, unpack_exhaustive_key
    rnd = random.Random(3)
    N, k_lo, k_hi = 696190560, 1, 8
    for _ in range(200):
        trip = [(rnd.randrange(1 << 29), rnd.randrange(N), rnd.randint(k_lo, k_hi)) for _ in range(5)]
        keys = [pack_exhaustive_key(T, r, k, N, k_lo, k_hi) for T, r, k in trip]
        assert max(keys) < (1 << 63)
        assert unpack_exhaustive_key(min(keys), N, k_lo, k_hi) == min(trip)
