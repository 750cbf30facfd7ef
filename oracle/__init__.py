"""CPU oracle for the AutoPipe planner/slicer hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package.  It shares no code with the
CUDA path; it is plain C (``autopipe_oracle.c``, gcc -O2) behind ctypes.  See that
file's header for the passage each function follows, and DESIGN.md §4 for the pins.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading
from concurrent.futures import ThreadPoolExecutor
from typing import Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "autopipe_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

OR_INF = (1 << 63) - 1


class OrOp(C.Structure):
    _fields_ = [("stage", C.c_int32), ("kind", C.c_int32), ("microbatch", C.c_int32),
                ("piece", C.c_int32), ("start_ns", C.c_int64), ("end_ns", C.c_int64)]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain -O2, no vectorisation pragmas)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = C.CDLL(_LIB)
            i32, i64, u64, u32 = C.c_int32, C.c_int64, C.c_uint64, C.c_uint32
            P = C.POINTER
            lib.or_comm_ns.restype = i64
            lib.or_comm_ns.argtypes = [i64, u64]
            lib.or_split.restype = i64
            lib.or_split.argtypes = [i64, i32, i32]
            lib.or_simulate_ex.restype = i32
            lib.or_simulate_ex.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, i32, i32,
                                           P(i32), P(i64), P(i32), P(OrOp), i32, P(i32),
                                           P(OrOp)]
            lib.or_num_ops.restype = i32
            lib.or_num_ops.argtypes = [i32, i32, i32, i32]
            lib.or_alg1.restype = i32
            lib.or_alg1.argtypes = [i32, P(i64), P(i64), i32, P(i32), P(i64)]
            lib.or_alg1_table.restype = None
            lib.or_alg1_table.argtypes = [i32, P(i64), P(i64), i32, P(i64), P(i32)]
            lib.or_alg1_reconstruct.restype = i32
            lib.or_alg1_reconstruct.argtypes = [P(i32), i32, i32, i32, i32, P(i32)]
            lib.or_min_lb.restype = i32
            lib.or_min_lb.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, i32, P(i64), P(i32)]
            lib.or_stage_feasible.restype = i32
            lib.or_stage_feasible.argtypes = [i32, P(i64), P(i64), i64, i32, i32, P(i32)]
            lib.or_exhaustive_mem.restype = i32
            lib.or_exhaustive_mem.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, i32, i32,
                                              P(i64), P(i64), i64, u64, u64, P(i64), P(u64),
                                              P(i32), P(i32), P(u64)]
            lib.or_count.restype = u64
            lib.or_count.argtypes = [i32, i32]
            lib.or_rank.restype = u64
            lib.or_rank.argtypes = [i32, i32, P(i32)]
            lib.or_unrank.restype = None
            lib.or_unrank.argtypes = [i32, i32, u64, P(i32)]
            lib.or_exhaustive.restype = i32
            lib.or_exhaustive.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, i32, i32,
                                          u64, u64, P(i64), P(u64), P(i32), P(i32), P(u64)]
            lib.or_lower_bound.restype = i64
            lib.or_lower_bound.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, i32, P(i32)]
            lib.or_exhaustive_bnb.restype = i32
            lib.or_exhaustive_bnb.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, i32, i32,
                                              i64, P(i64), P(u64), P(i32), P(i32), P(u64),
                                              P(u64)]
            lib.or_splitmix64.restype = u64
            lib.or_splitmix64.argtypes = [u64]
            lib.or_restart_start.restype = None
            lib.or_restart_start.argtypes = [i32, i32, P(i32), u64, i32, u32, P(i32)]
            lib.or_heuristic_restart.restype = i32
            lib.or_heuristic_restart.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, u64,
                                                 i32, u32, P(i64), P(i32), P(u64), P(i32)]
            lib.or_heuristic.restype = i32
            lib.or_heuristic.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, u64, i32, u32,
                                         u32, P(i64), P(u32), P(i32), P(i64), P(u64)]
            lib.or_heuristic_ex.restype = i32
            lib.or_heuristic_ex.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, u64, i32, u32,
                                            u32, i32, P(i64), P(u32), P(i32), P(i64), P(u64)]
            lib.or_reach_restart.restype = i32
            lib.or_reach_restart.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, u64, i32, u32,
                                             i32, P(i64), P(i32), P(u64), P(i32)]
            lib.or_reach.restype = i32
            lib.or_reach.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, u64, i32, u32, u32,
                                     i32, P(i64), P(u32), P(i32), P(u64), P(u32)]
            lib.or_heuristic_restart_ex.restype = i32
            lib.or_heuristic_restart_ex.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, u64,
                                                    i32, u32, i32, P(i64), P(i32), P(u64), P(i32)]
            lib.or_slice_sweep_paper.restype = i32
            lib.or_slice_sweep_paper.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, P(i32),
                                                 i32, i32, P(i64), P(i32)]
            lib.or_alg2.restype = i32
            lib.or_alg2.argtypes = [i32, P(i64), P(i64), P(i64), i32, P(i32), i32, P(i32)]
            lib.or_alg2_trace.restype = i32
            lib.or_alg2_trace.argtypes = [i32, P(i64), P(i64), P(i64), i32, P(i32), i32, P(i32),
                                          P(i64), P(i64), P(i64)]
            lib.or_slice_sweep.restype = i32
            lib.or_slice_sweep.argtypes = [i32, P(i64), P(i64), P(i64), i32, i32, P(i32), i32,
                                           P(i64), P(i32)]
            _lib = lib
    return _lib


def _i64(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int64))


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def _p(a, ct):
    return a.ctypes.data_as(C.POINTER(ct))


class OracleError(RuntimeError):
    pass


def _chk(rc):
    if rc != 0:
        raise OracleError(f"oracle status {rc}")


class Model:
    """Per-sub-layer tables plus the derived comm_ns vector (oracle-side)."""

    def __init__(self, fwd_ns, bwd_ns, act_bytes, link_bytes_per_s: int):
        self.f = _i64(fwd_ns)
        self.b = _i64(bwd_ns)
        self.act = _i64(act_bytes)
        self.bw = int(link_bytes_per_s)
        self.n = int(self.f.shape[0])
        lib = _load()
        self.comm = _i64([lib.or_comm_ns(int(self.act[i]), self.bw) for i in range(self.n)])

    @classmethod
    def from_workload(cls, wl) -> "Model":
        return cls(wl.fwd_ns, wl.bwd_ns, wl.act_bytes, wl.link_bytes_per_s)

    # ------------------------------------------------------------------ sim
    def simulate(self, p: int, m: int, cuts, k: int = 1, s: int = 1,
                 want_path: bool = False, want_all: bool = False):
        """Returns dict(T, master[, path][, ops])."""
        lib = _load()
        c = _i32(cuts)
        T = C.c_int64(); master = C.c_int32(); L = C.c_int32()
        nops = lib.or_num_ops(p, m, s, k)
        cap = nops
        path = (OrOp * cap)() if want_path else None
        allops = (OrOp * nops)() if want_all else None
        rc = lib.or_simulate_ex(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                _p(self.comm, C.c_int64), p, m, s, k, _p(c, C.c_int32),
                                C.byref(T), C.byref(master), path, cap, C.byref(L), allops)
        _chk(rc)
        out = {"T": T.value, "master": master.value, "path_len": L.value}
        if want_path:
            out["path"] = [(o.stage, o.kind, o.microbatch, o.piece, o.start_ns, o.end_ns)
                           for o in path[:L.value]]
        if want_all:
            out["ops"] = [(o.stage, o.kind, o.microbatch, o.piece, o.start_ns, o.end_ns)
                          for o in allops[:nops]]
        return out

    def T(self, p, m, cuts, k=1, s=1) -> int:
        return self.simulate(p, m, cuts, k=k, s=s)["T"]

    # ------------------------------------------------------------- alg. 1
    def alg1(self, p: int):
        lib = _load()
        cuts = np.zeros(max(p - 1, 1), np.int32); v = C.c_int64()
        _chk(lib.or_alg1(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64), p,
                         _p(cuts, C.c_int32), C.byref(v)))
        return cuts[: p - 1].copy(), v.value

    def alg1_table(self, p: int):
        lib = _load()
        P = min(p, self.n)
        t = np.zeros((self.n + 1, P + 1), np.int64)
        a = np.zeros((self.n + 1, P + 1), np.int32)
        lib.or_alg1_table(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64), p,
                          _p(t, C.c_int64), _p(a, C.c_int32))
        return t, a

    # --------------------------------------------------------- exhaustive
    def exhaustive(self, p, m, k_lo=1, k_hi=1, rank_lo=0, rank_hi=None):
        lib = _load()
        if rank_hi is None:
            rank_hi = count(self.n, p)
        T = C.c_int64(); r = C.c_uint64(); k = C.c_int32(); sims = C.c_uint64()
        cuts = np.zeros(max(p - 1, 1), np.int32)
        _chk(lib.or_exhaustive(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                               _p(self.comm, C.c_int64), p, m, k_lo, k_hi, rank_lo, rank_hi,
                               C.byref(T), C.byref(r), C.byref(k), _p(cuts, C.c_int32),
                               C.byref(sims)))
        return {"T": T.value, "rank": r.value, "k": k.value, "cuts": cuts[: p - 1].copy(),
                "sims": sims.value}

    def exhaustive_parallel(self, p, m, k_lo=1, k_hi=1, rank_lo=0, rank_hi=None,
                            threads: Optional[int] = None):
        """Same result as exhaustive(): contiguous rank ranges on host threads (the
        C code releases the GIL), combined by min (T, rank, k)."""
        if rank_hi is None:
            rank_hi = count(self.n, p)
        threads = threads or os.cpu_count() or 1
        tot = rank_hi - rank_lo
        edges = [rank_lo + (tot * i) // threads for i in range(threads + 1)]
        with ThreadPoolExecutor(threads) as ex:
            res = list(ex.map(lambda i: self.exhaustive(p, m, k_lo, k_hi, edges[i], edges[i + 1]),
                              [i for i in range(threads) if edges[i + 1] > edges[i]]))
        best = min(res, key=lambda d: (d["T"], d["rank"], d["k"]))
        best = dict(best)
        best["sims"] = sum(d["sims"] for d in res)
        return best

    # ------------------------------------------------- N4 depth + memory (R-N4)
    def feasible(self, p, m, cuts, static_bytes, stash_bytes, cap) -> bool:
        lib = _load()
        c = _i32(cuts) if p > 1 else np.zeros(1, np.int32)
        return bool(lib.or_stage_feasible(self.n, _p(_i64(static_bytes), C.c_int64),
                                          _p(_i64(stash_bytes), C.c_int64), int(cap), p, m,
                                          _p(c, C.c_int32)))

    def exhaustive_mem(self, p, m, k_lo, k_hi, static_bytes, stash_bytes, cap, rank_lo=0,
                       rank_hi=None):
        """Exhaustive argmin over the memory-feasible partitions; T = None if none."""
        lib = _load()
        if rank_hi is None:
            rank_hi = count(self.n, p)
        T = C.c_int64(); r = C.c_uint64(); k = C.c_int32(); sims = C.c_uint64()
        cuts = np.zeros(max(p - 1, 1), np.int32)
        sb, tb = _i64(static_bytes), _i64(stash_bytes)
        _chk(lib.or_exhaustive_mem(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                   _p(self.comm, C.c_int64), p, m, k_lo, k_hi,
                                   _p(sb, C.c_int64), _p(tb, C.c_int64), int(cap),
                                   int(rank_lo), int(rank_hi), C.byref(T), C.byref(r), C.byref(k), _p(cuts, C.c_int32),
                                   C.byref(sims)))
        if T.value == (1 << 63) - 1:
            return {"T": None, "sims": sims.value}
        return {"T": T.value, "rank": r.value, "k": k.value, "cuts": cuts[: p - 1].copy(),
                "sims": sims.value}

    def plan_depths(self, n_gpus, microbatches, static_bytes, stash_bytes, cap, k_lo=1, k_hi=1):
        """Outer planner loop (NEXT N4, reading R-N4): every depth p dividing n_gpus
        (p <= n) whose data-parallel width dp = n_gpus/p divides `microbatches`;
        m = microbatches/dp; the feasible argmin per p; best = least (T, p)."""
        per = []
        for p in range(1, min(self.n, n_gpus) + 1):
            if n_gpus % p or microbatches % (n_gpus // p):
                continue
            m = microbatches // (n_gpus // p)
            r = self.exhaustive_mem(p, m, k_lo, k_hi, static_bytes, stash_bytes, cap)
            r.update({"p": p, "m": m, "dp": n_gpus // p})
            per.append(r)
        feas = [r for r in per if r["T"] is not None]
        best = min(feas, key=lambda r: (r["T"], r["p"])) if feas else None
        return best, per

    def lower_bound(self, p, m, K, cuts) -> int:
        lib = _load()
        c = _i32(cuts)
        return lib.or_lower_bound(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                  _p(self.comm, C.c_int64), p, m, K, _p(c, C.c_int32))

    def min_lower_bound(self, p, m, K=1):
        """Certified minLB over all partitions and k <= K (DESIGN.md
        reading R-LB): returns (lb, cuts of an argmin partition of the relaxed bound)."""
        lib = _load()
        lb = C.c_int64()
        cuts = np.zeros(max(p - 1, 1), np.int32)
        _chk(lib.or_min_lb(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                           _p(self.comm, C.c_int64), p, m, K, C.byref(lb), _p(cuts, C.c_int32)))
        return lb.value, cuts[: p - 1].copy()

    def exhaustive_bnb(self, p, m, k_lo=1, k_hi=1, incumbent: Optional[int] = None):
        lib = _load()
        if incumbent is None:
            cuts0, _ = self.alg1(p)
            incumbent = self.T(p, m, cuts0, k=k_lo)
        T = C.c_int64(); r = C.c_uint64(); k = C.c_int32(); sims = C.c_uint64()
        leaves = C.c_uint64()
        cuts = np.zeros(max(p - 1, 1), np.int32)
        _chk(lib.or_exhaustive_bnb(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                   _p(self.comm, C.c_int64), p, m, k_lo, k_hi, incumbent,
                                   C.byref(T), C.byref(r), C.byref(k), _p(cuts, C.c_int32),
                                   C.byref(sims), C.byref(leaves)))
        return {"T": T.value, "rank": r.value, "k": k.value, "cuts": cuts[: p - 1].copy(),
                "sims": sims.value, "leaves": leaves.value, "incumbent": incumbent}

    # ---------------------------------------------------------- heuristic
    def restart_start(self, p, seed, radius, r):
        lib = _load()
        a1, _ = self.alg1(p)
        a1 = _i32(a1) if p > 1 else np.zeros(1, np.int32)
        out = np.zeros(max(p - 1, 1), np.int32)
        lib.or_restart_start(self.n, p, _p(a1, C.c_int32), seed, radius, r, _p(out, C.c_int32))
        return out[: p - 1].copy()

    def heuristic_restart(self, p, m, seed, radius, r, adjust_mode: int = 0):
        lib = _load()
        T = C.c_int64(); sims = C.c_uint64(); steps = C.c_int32()
        cuts = np.zeros(max(p - 1, 1), np.int32)
        _chk(lib.or_heuristic_restart_ex(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                         _p(self.comm, C.c_int64), p, m, seed, radius, r,
                                         adjust_mode, C.byref(T), _p(cuts, C.c_int32),
                                         C.byref(sims), C.byref(steps)))
        return {"T": T.value, "cuts": cuts[: p - 1].copy(), "sims": sims.value,
                "steps": steps.value}

    def heuristic(self, p, m, seed, radius, r_lo, r_hi, per_restart: bool = False,
                  adjust_mode: int = 0):
        lib = _load()
        T = C.c_int64(); r = C.c_uint32(); sims = C.c_uint64()
        cuts = np.zeros(max(p - 1, 1), np.int32)
        per = np.zeros(max(r_hi - r_lo, 1), np.int64)
        _chk(lib.or_heuristic_ex(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                 _p(self.comm, C.c_int64), p, m, seed, radius, r_lo, r_hi,
                                 adjust_mode, C.byref(T), C.byref(r), _p(cuts, C.c_int32),
                                 _p(per, C.c_int64), C.byref(sims)))
        out = {"T": T.value, "restart": r.value, "cuts": cuts[: p - 1].copy(), "sims": sims.value}
        if per_restart:
            out["per_restart_T"] = per[: r_hi - r_lo].copy()
        return out

    def reach_restart(self, p, m, seed, radius, r, vmax=4096):
        """Reachable-set search of one restart (NEXT N1, reading R-N1)."""
        lib = _load()
        T = C.c_int64(); sims = C.c_uint64(); tr = C.c_int32()
        cuts = np.zeros(max(p - 1, 1), np.int32)
        _chk(lib.or_reach_restart(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                  _p(self.comm, C.c_int64), p, m, seed, radius, r, vmax,
                                  C.byref(T), _p(cuts, C.c_int32), C.byref(sims), C.byref(tr)))
        return {"T": T.value, "cuts": cuts[: p - 1].copy(), "sims": sims.value,
                "truncated": bool(tr.value)}

    def reach(self, p, m, seed, radius, r_lo, r_hi, vmax=4096):
        lib = _load()
        T = C.c_int64(); r = C.c_uint32(); sims = C.c_uint64(); tr = C.c_uint32()
        cuts = np.zeros(max(p - 1, 1), np.int32)
        _chk(lib.or_reach(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                          _p(self.comm, C.c_int64), p, m, seed, radius, r_lo, r_hi, vmax,
                          C.byref(T), C.byref(r), _p(cuts, C.c_int32), C.byref(sims),
                          C.byref(tr)))
        return {"T": T.value, "restart": r.value, "cuts": cuts[: p - 1].copy(),
                "sims": sims.value, "truncated": tr.value}

    def reach_parallel(self, p, m, seed, radius, r_lo, r_hi, vmax=4096, threads=None):
        threads = threads or os.cpu_count() or 1
        tot = r_hi - r_lo
        edges = [r_lo + (tot * i) // threads for i in range(threads + 1)]
        idx = [i for i in range(threads) if edges[i + 1] > edges[i]]
        with ThreadPoolExecutor(threads) as ex:
            res = list(ex.map(lambda i: self.reach(p, m, seed, radius, edges[i], edges[i + 1],
                                                   vmax), idx))
        best = dict(min(res, key=lambda d: (d["T"], d["restart"])))
        best["sims"] = sum(d["sims"] for d in res)
        best["truncated"] = sum(d["truncated"] for d in res)
        return best

    def heuristic_parallel(self, p, m, seed, radius, r_lo, r_hi, threads=None,
                           per_restart: bool = False, adjust_mode: int = 0):
        threads = threads or os.cpu_count() or 1
        tot = r_hi - r_lo
        edges = [r_lo + (tot * i) // threads for i in range(threads + 1)]
        idx = [i for i in range(threads) if edges[i + 1] > edges[i]]
        with ThreadPoolExecutor(threads) as ex:
            res = list(ex.map(lambda i: self.heuristic(p, m, seed, radius, edges[i], edges[i + 1],
                                                       per_restart, adjust_mode), idx))
        best = dict(min(res, key=lambda d: (d["T"], d["restart"])))
        best["sims"] = sum(d["sims"] for d in res)
        if per_restart:
            best["per_restart_T"] = np.concatenate([d["per_restart_T"] for d in res])
        return best

    def slice_sweep(self, p, m, cuts, K):
        lib = _load()
        c = _i32(cuts)
        T = np.zeros(K, np.int64); bk = C.c_int32()
        _chk(lib.or_slice_sweep(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                _p(self.comm, C.c_int64), p, m, _p(c, C.c_int32), K,
                                _p(T, C.c_int64), C.byref(bk)))
        return T, bk.value


def _slice_paper(self, p, m, cuts, k, s_max):
    lib = _load()
    c = _i32(cuts) if p > 1 else np.zeros(1, np.int32)
    T = np.zeros(s_max + 1, np.int64); bs = C.c_int32()
    _chk(lib.or_slice_sweep_paper(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                                  _p(self.comm, C.c_int64), p, m, _p(c, C.c_int32), k, s_max,
                                  _p(T, C.c_int64), C.byref(bs)))
    return T, bs.value


def _alg2(self, p, cuts, reading=0):
    lib = _load()
    c = _i32(cuts) if p > 1 else np.zeros(1, np.int32)
    mb = C.c_int32()
    _chk(lib.or_alg2(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                     _p(self.comm, C.c_int64), p, _p(c, C.c_int32), reading, C.byref(mb)))
    return mb.value


def _alg2_trace(self, p, cuts, reading=0):
    """Algorithm 2 with its state recorded (see or_alg2_trace): returns
    (mb, startt[p], [endt rows per pass], [tempt per pass])."""
    lib = _load()
    c = _i32(cuts) if p > 1 else np.zeros(1, np.int32)
    mb = C.c_int32()
    st = np.zeros(p, np.int64)
    en = np.zeros(p * (p + 1) * 2, np.int64)
    te = np.zeros(p, np.int64)
    _chk(lib.or_alg2_trace(self.n, _p(self.f, C.c_int64), _p(self.b, C.c_int64),
                           _p(self.comm, C.c_int64), p, _p(c, C.c_int32), reading, C.byref(mb),
                           _p(st, C.c_int64), _p(en, C.c_int64), _p(te, C.c_int64)))
    en = en.reshape(p, p + 1, 2)
    return (mb.value, [int(x) for x in st],
            [[[int(v) for v in row] for row in en[i]] for i in range(mb.value)],
            [int(x) for x in te[: mb.value]])


Model.slice_sweep_paper = _slice_paper
Model.alg2 = _alg2
Model.alg2_trace = _alg2_trace


def count(n: int, p: int) -> int:
    return int(_load().or_count(n, p))


def rank(n: int, p: int, cuts) -> int:
    c = _i32(cuts)
    return int(_load().or_rank(n, p, _p(c, C.c_int32)))


def unrank(n: int, p: int, r: int):
    c = np.zeros(max(p - 1, 1), np.int32)
    _load().or_unrank(n, p, r, _p(c, C.c_int32))
    return [int(x) for x in c[: p - 1]]


def comm_ns(nbytes: int, bw: int) -> int:
    return int(_load().or_comm_ns(nbytes, bw))


def split(v: int, k: int, q: int) -> int:
    return int(_load().or_split(v, k, q))


def splitmix64(s: int) -> int:
    return int(_load().or_splitmix64(s))
