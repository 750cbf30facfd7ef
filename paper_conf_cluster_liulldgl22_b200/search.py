"""Multi-GPU search orchestration (one process per GPU, torch.distributed/NCCL).

The candidate space is sharded by contiguous lex-rank (or restart) ranges
``[floor(g*N/G), floor((g+1)*N/G))`` -- SURVEY.md §8e.  Each rank writes one packed
int64 key on its GPU; ONE ``all_reduce(MIN)`` of that 8-byte key over NVLink picks
the global winner, which every rank then decodes independently (no second
collective).  The reduction is exact because keys order lexicographically by
(T, rank, k) / (T, restart) -- include/ap.h.  When T << rb | index does not fit in
63 bits, the two-phase form (NEXT N3) reduces T first and then the least index among
the ranks holding T*: two 8-byte all-reduces instead of one.
"""
from __future__ import annotations

from typing import Optional

import torch

from . import (AP_ERR_RANGE, AP_KEY_RANGE, AP_SEARCH_MEMORY, INT64_MAX, APError, Plan, ap_count, ap_decode,
               ap_key2_select, ap_search_exhaustive, ap_search_exhaustive2,
               ap_search_heuristic)


def shard(total: int, rank: int, world: int):
    """Contiguous [lo, hi) slice of `total` units for `rank` of `world`."""
    return (total * rank) // world, (total * (rank + 1)) // world


def rank_bits(N: int, K: int) -> int:
    """rb = bitlen(N*K - 1): low bits of an exhaustive key (include/ap.h)."""
    return (N * K - 1).bit_length()


def pack_exhaustive_key(T: int, rank: int, k: int, N: int, k_lo: int, k_hi: int) -> int:
    """key = T << rb | (rank*K + k - k_lo) -- the layout ap_search_exhaustive writes."""
    K = k_hi - k_lo + 1
    return (T << rank_bits(N, K)) | (rank * K + k - k_lo)


def unpack_exhaustive_key(key: int, N: int, k_lo: int, k_hi: int):
    """(T, rank, k) of a reduced exhaustive key; None for INT64_MAX (empty)."""
    if key == INT64_MAX:
        return None
    K = k_hi - k_lo + 1
    rb = rank_bits(N, K)
    idx = key & ((1 << rb) - 1)
    return key >> rb, idx // K, k_lo + idx % K


def unpack_heuristic_key(key: int):
    """(T, restart) of a reduced heuristic key (T << 20 | r)."""
    if key == INT64_MAX:
        return None
    return key >> 20, key & ((1 << 20) - 1)


def _world():
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        return dist.get_rank(), dist.get_world_size(), dist
    return 0, 1, None


def min_allreduce_key(key: torch.Tensor, dist=None, group=None) -> torch.Tensor:
    """In-place MIN all-reduce of the packed int64 key (no-op on one process)."""
    if dist is not None:
        dist.all_reduce(key, op=dist.ReduceOp.MIN, group=group)
    return key


def two_phase_reduce(local: torch.Tensor, dist=None, group=None, select=None):
    """Two-phase MIN reduction of per-rank (T, index) pairs (int64[2] tensors):
    T* = min T; index = min over the ranks whose T == T* (the others contribute
    INT64_MAX through `select`, default the device kernel ap_key2_select).
    Returns (T*, index) as Python ints."""
    select = select or (lambda loc, ts, idx: ap_key2_select(loc, ts, idx))
    t_star = local[:1].clone()
    min_allreduce_key(t_star, dist, group)
    idx = torch.empty(1, dtype=torch.int64, device=local.device)
    select(local, t_star, idx)
    min_allreduce_key(idx, dist, group)
    return int(t_star.item()), int(idx.item())


def search_exhaustive(plan: Plan, p: int, m: int, k_lo: int = 1, k_hi: int = 1,
                      group=None, decode: bool = True, stream=None,
                      two_phase: Optional[bool] = None, mode: int = 0) -> dict:
    """Exact argmin over all C(n-1,p-1) partitions x k in [k_lo,k_hi], sharded over
    the ranks of the default process group (if initialised).  two_phase None: the
    packed key when it fits, else the two-phase reduction.  The packing test needs T_ref,
    which only the device knows: a search whose key does not fit writes AP_KEY_RANGE (the
    least int64), the MIN all-reduce hands it to every rank (an empty shard included),
    and all ranks then run the two-phase form together."""
    rank, world, dist = _world()
    N = ap_count(plan.n, p)
    lo, hi = shard(N, rank, world)
    dev = f"cuda:{plan.device}"
    out = {"sims": (hi - lo) * (k_hi - k_lo + 1), "total_sims": N * (k_hi - k_lo + 1),
           "shard": (lo, hi), "two_phase": False}
    if not two_phase:
        key = torch.empty(1, dtype=torch.int64, device=dev)
        if hi > lo:
            from . import ap_search_exhaustive_mode
            ap_search_exhaustive_mode(plan, p, m, k_lo, k_hi, lo, hi, mode, key, stream=stream)
        else:
            key.fill_(INT64_MAX)
        min_allreduce_key(key, dist, group)
        kv = int(key.item())
        if kv == AP_KEY_RANGE:
            # T_ref << rb does not fit (decided on the device); the MIN reduction handed
            # the sentinel to every rank, empty shards included, so all switch together
            if two_phase is not None:
                raise APError(AP_ERR_RANGE, "key packing: the packed key does not fit")
            two_phase = True
        else:
            out["key"] = kv
            if decode and kv != INT64_MAX:
                out.update(ap_decode(plan, 0, p, m, k_lo, k_hi, key=kv))
            return out
    local = torch.empty(2, dtype=torch.int64, device=dev)
    if hi > lo:
        ap_search_exhaustive2(plan, p, m, k_lo, k_hi, lo, hi, mode, local, stream=stream)
    else:
        local.fill_(INT64_MAX)
    T, idx = two_phase_reduce(local, dist, group)
    out.update({"two_phase": True, "key": idx, "T": T})
    if decode and idx != INT64_MAX:
        res = ap_decode(plan, 2, p, m, k_lo, k_hi, key=idx)
        if res["time_ns"] != T:
            raise RuntimeError(f"two-phase decode: T*={T}, re-simulated {res['time_ns']}")
        out.update(res)
    return out


def plan_pipeline_depth(plan: Plan, n_gpus: int, microbatches: int, k_lo: int = 1,
                        k_hi: int = 1, group=None) -> dict:
    """NEXT N4 (reading R-N4): the outer planner loop over pipeline depth.
    Needs ap_plan_set_memory on `plan`.  For every depth p dividing n_gpus (p <= n,
    <= AP_MAX_P) whose data-parallel width dp = n_gpus / p divides `microbatches`:
    m = microbatches / dp, and the exact argmin over the memory-feasible partitions
    (AP_SEARCH_MEMORY, sharded over the ranks like search_exhaustive).  The plan is the
    least (T, p); no data-parallel all-reduce term (reading Q12)."""
    from . import AP_MAX_P
    per = []
    for p in range(1, min(plan.n, n_gpus, AP_MAX_P) + 1):
        if n_gpus % p or microbatches % (n_gpus // p):
            continue
        m = microbatches // (n_gpus // p)
        r = search_exhaustive(plan, p, m, k_lo, k_hi, group=group, decode=False,
                              mode=AP_SEARCH_MEMORY)
        row = {"p": p, "dp": n_gpus // p, "m": m, "two_phase": r["two_phase"],
               "sims": r["total_sims"]}
        key = r["key"]
        if key == INT64_MAX:
            row["T"] = None
        else:
            res = ap_decode(plan, 2 if r["two_phase"] else 0, p, m, k_lo, k_hi, key=key)
            row.update({"T": res["time_ns"], "rank": res["rank"], "k": res["k"],
                        "cuts": res["cuts"], "master": res["master"]})
        per.append(row)
    feas = [r for r in per if r["T"] is not None]
    best = min(feas, key=lambda r: (r["T"], r["p"])) if feas else None
    return {"best": best, "per_depth": per}


def search_heuristic(plan: Plan, p: int, m: int, restarts: int, seed: int = 0x5EED,
                     radius: int = 2, group=None, decode: bool = True, stream=None) -> dict:
    rank, world, dist = _world()
    lo, hi = shard(restarts, rank, world)
    key = torch.empty(1, dtype=torch.int64, device=f"cuda:{plan.device}")
    if hi > lo:
        ap_search_heuristic(plan, p, m, seed, radius, lo, hi, 0, key, stream=stream)
    else:
        key.fill_(INT64_MAX)
    min_allreduce_key(key, dist, group)
    kv = int(key.item())
    out = {"key": kv, "shard": (lo, hi)}
    if decode:
        out.update(ap_decode(plan, 1, p, m, seed=seed, radius=radius, key=kv))
    return out
