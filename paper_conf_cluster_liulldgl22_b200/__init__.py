"""B200-native AutoPipe planner/slicer hot path -- thin Python binding of include/ap.h.

Every function here has the name of the C-ABI call it wraps and only marshals
arguments (torch device tensors -> raw pointers, the current CUDA stream -> the
stream handle).  All computation happens in libap.so's sm_100a kernels; if the
library is missing this module raises at import time -- there is no fallback.

Higher-level helpers (multi-GPU sharding + NCCL min-all-reduce) are in
``paper_conf_cluster_liulldgl22_b200.search``.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("AP_LIB_PATH") or os.path.join(_HERE, "libap.so")

AP_MAX_P = 32
AP_MAX_K = 16
AP_MAX_N = 512
INT64_MAX = (1 << 63) - 1
AP_KEY_RANGE = -(1 << 63)  # include/ap.h: packed exhaustive key that does not fit
AP_OK, AP_ERR_INVALID, AP_ERR_RANGE, AP_ERR_CUDA, AP_ERR_NOMEM, AP_ERR_CAPACITY = range(6)

_STATUS = {0: "AP_OK", 1: "AP_ERR_INVALID", 2: "AP_ERR_RANGE", 3: "AP_ERR_CUDA",
           4: "AP_ERR_NOMEM", 5: "AP_ERR_CAPACITY"}


class APError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class ApResult(C.Structure):
    _fields_ = [("time_ns", C.c_int64), ("rank", C.c_uint64), ("restart", C.c_uint32),
                ("k", C.c_int32), ("master", C.c_int32), ("p", C.c_int32),
                ("cuts", C.c_int32 * (AP_MAX_P - 1))]


class ApOp(C.Structure):
    _fields_ = [("stage", C.c_int32), ("kind", C.c_int32), ("microbatch", C.c_int32),
                ("piece", C.c_int32), ("start_ns", C.c_int64), ("end_ns", C.c_int64)]


class ApLaunchInfo(C.Structure):
    _fields_ = [("fast_u32", C.c_int32), ("exact_p", C.c_int32), ("blocks", C.c_int32),
                ("threads", C.c_int32), ("chunk", C.c_uint64), ("t_ref", C.c_int64),
                ("rank_bits", C.c_int32), ("launches", C.c_int32), ("clamp_rows", C.c_int32),
                ("clamp_first", C.c_int32), ("clamp_final", C.c_int32)]


def _load_lib():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built; run __graft_entry__.build() "
                          "(there is no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    i32, i64, u64, u32, vp = C.c_int32, C.c_int64, C.c_uint64, C.c_uint32, C.c_void_p
    P = C.POINTER
    lib.ap_last_error.restype = C.c_char_p
    lib.ap_version.restype = C.c_char_p
    lib.ap_plan_create.restype = i32
    lib.ap_plan_create.argtypes = [i32, P(i64), P(i64), P(i64), u64, i32, P(vp)]
    lib.ap_plan_destroy.restype = None
    lib.ap_plan_destroy.argtypes = [vp]
    lib.ap_plan_info.restype = i32
    lib.ap_plan_info.argtypes = [vp, P(i32), P(i64)]
    lib.ap_count.restype = i32
    lib.ap_count.argtypes = [i32, i32, P(u64)]
    lib.ap_eval_batch.restype = i32
    lib.ap_eval_batch.argtypes = [vp, i32, i32, vp, vp, i64, vp, vp, vp]
    lib.ap_eval_batch_ex.restype = i32
    lib.ap_eval_batch_ex.argtypes = [vp, i32, i32, vp, vp, i64, vp, vp, vp, vp]
    lib.ap_search_exhaustive.restype = i32
    lib.ap_search_exhaustive.argtypes = [vp, i32, i32, i32, i32, u64, u64, vp, vp]
    lib.ap_search_exhaustive_mode.restype = i32
    lib.ap_search_exhaustive_mode.argtypes = [vp, i32, i32, i32, i32, u64, u64, i32, vp, vp]
    lib.ap_search_heuristic.restype = i32
    lib.ap_search_heuristic.argtypes = [vp, i32, i32, u64, i32, u32, u32, i32, vp, vp]
    lib.ap_decode.restype = i32
    lib.ap_decode.argtypes = [vp, i32, i32, i32, i32, i32, u64, i32, i32, i64, P(ApResult)]
    lib.ap_slice_sweep.restype = i32
    lib.ap_slice_sweep.argtypes = [vp, i32, i32, P(i32), i32, P(i64), P(i32)]
    lib.ap_slice_sweep_paper.restype = i32
    lib.ap_slice_sweep_paper.argtypes = [vp, i32, i32, P(i32), i32, i32, P(i64), P(i32)]
    lib.ap_slicer_alg2.restype = i32
    lib.ap_slicer_alg2.argtypes = [vp, i32, P(i32), i32, P(i32)]
    lib.ap_critical_path.restype = i32
    lib.ap_critical_path.argtypes = [vp, i32, i32, i32, P(i32), P(ApOp), i32, P(i32), P(i32),
                                     P(i64)]
    lib.ap_alg1.restype = i32
    lib.ap_alg1.argtypes = [vp, i32, P(i32), P(i64)]
    lib.ap_search_exhaustive2.restype = i32
    lib.ap_search_exhaustive2.argtypes = [vp, i32, i32, i32, i32, u64, u64, i32, vp, vp]
    lib.ap_search_exhaustive_bounded.restype = i32
    lib.ap_search_exhaustive_bounded.argtypes = [vp, i32, i32, i32, i32, u64, u64, i32, i64, vp, vp]
    lib.ap_key2_select.restype = i32
    lib.ap_key2_select.argtypes = [vp, vp, vp, vp]
    lib.ap_search_reachable.restype = i32
    lib.ap_search_reachable.argtypes = [vp, i32, i32, u64, i32, u32, u32, i32, vp, vp]
    lib.ap_decode_reachable.restype = i32
    lib.ap_decode_reachable.argtypes = [vp, i32, i32, u64, i32, i32, i64, P(ApResult)]
    lib.ap_last_truncated.restype = i32
    lib.ap_last_truncated.argtypes = [P(u64)]
    lib.ap_plan_set_memory.restype = i32
    lib.ap_plan_set_memory.argtypes = [vp, P(i64), P(i64), i64]
    lib.ap_min_lower_bound.restype = i32
    lib.ap_min_lower_bound.argtypes = [vp, i32, i32, i32, P(i64), P(i32)]
    lib.ap_last_launch.restype = None
    lib.ap_last_launch.argtypes = [P(ApLaunchInfo)]
    lib.ap_last_kernel_ms.restype = i32
    lib.ap_last_kernel_ms.argtypes = [P(C.c_float)]
    lib.ap_last_sims.restype = i32
    lib.ap_last_sims.argtypes = [P(u64)]
    lib.ap_kernel_launches.restype = u64
    lib.ap_kernel_launches.argtypes = []
    return lib


lib = _load_lib()

# every symbol include/ap.h declares (checked by tests/test_abi.py)
EXPORTS = ("ap_last_error", "ap_version", "ap_plan_create", "ap_plan_destroy", "ap_plan_info",
           "ap_plan_set_memory",
           "ap_count", "ap_eval_batch", "ap_eval_batch_ex", "ap_search_exhaustive", "ap_search_exhaustive_mode",
           "ap_search_exhaustive2", "ap_search_exhaustive_bounded", "ap_key2_select",
           "ap_search_heuristic", "ap_search_reachable", "ap_decode_reachable",
           "ap_last_truncated",
           "ap_decode", "ap_slice_sweep", "ap_slice_sweep_paper", "ap_slicer_alg2",
           "ap_critical_path", "ap_alg1", "ap_min_lower_bound", "ap_last_launch",
           "ap_last_kernel_ms", "ap_last_sims", "ap_kernel_launches")


def _check(st: int):
    if st != 0:
        raise APError(st, lib.ap_last_error().decode())


def _i64(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int64))


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def _ptr(t, dtype_name: str, device_index: Optional[int] = None, min_numel: int = 0):
    """data_ptr of a contiguous CUDA torch tensor of the given dtype (or None)."""
    if t is None:
        return None
    import torch
    want = {"int32": torch.int32, "int64": torch.int64}[dtype_name]
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError("expected a CUDA torch tensor")
    if t.dtype != want or not t.is_contiguous():
        raise TypeError(f"expected a contiguous {dtype_name} tensor, got {t.dtype}")
    if device_index is not None and t.device.index != device_index:
        raise ValueError(f"tensor on cuda:{t.device.index}, plan on cuda:{device_index}")
    if t.numel() < min_numel:
        raise ValueError(f"expected at least {min_numel} elements, got {t.numel()}")
    return C.c_void_p(t.data_ptr())


def _stream(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


class Plan:
    """Owning handle for an ``ap_plan``."""

    def __init__(self, handle: int, n: int, device: int):
        self._h = C.c_void_p(handle)
        self.n = n
        self.device = device

    @property
    def handle(self):
        return self._h

    def comm_ns(self) -> np.ndarray:
        out = np.zeros(self.n, np.int64)
        nn = C.c_int32()
        _check(lib.ap_plan_info(self._h, C.byref(nn), out.ctypes.data_as(C.POINTER(C.c_int64))))
        return out

    def close(self):
        if self._h is not None and self._h.value:
            lib.ap_plan_destroy(self._h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def ap_version() -> str:
    return lib.ap_version().decode()


def ap_last_error() -> str:
    return lib.ap_last_error().decode()


def ap_plan_create(fwd_ns, bwd_ns, act_bytes, link_bytes_per_s: int, device: int = 0) -> Plan:
    f, b, a = _i64(fwd_ns), _i64(bwd_ns), _i64(act_bytes)
    if not (f.shape == b.shape == a.shape) or f.ndim != 1:
        raise ValueError("fwd_ns, bwd_ns, act_bytes must be 1-D of equal length")
    h = C.c_void_p()
    P = C.POINTER(C.c_int64)
    _check(lib.ap_plan_create(int(f.shape[0]), f.ctypes.data_as(P), b.ctypes.data_as(P),
                              a.ctypes.data_as(P), int(link_bytes_per_s), int(device),
                              C.byref(h)))
    return Plan(h.value, int(f.shape[0]), int(device))


def ap_plan_destroy(plan: Plan) -> None:
    plan.close()


def ap_count(n: int, p: int) -> int:
    out = C.c_uint64()
    _check(lib.ap_count(int(n), int(p), C.byref(out)))
    return out.value


def ap_eval_batch(plan: Plan, p: int, m: int, cuts, k, time_ns, master=None, stream=None,
                  n_invalid=None):
    """cuts: int32 CUDA [count, p-1]; k: int32 CUDA [count] or None; time_ns: int64
    CUDA [count] (written); master: int32 CUDA [count] or None; n_invalid: int64 CUDA [1]
    or None (ap_eval_batch_ex: receives the number of invalid rows, which read -1).
    Asynchronous."""
    count = int(time_ns.numel())
    args = (plan.handle, int(p), int(m), _ptr(cuts, "int32", plan.device),
            _ptr(k, "int32", plan.device), count, _ptr(time_ns, "int64", plan.device),
            _ptr(master, "int32", plan.device))
    if n_invalid is None:
        _check(lib.ap_eval_batch(*args, _stream(stream)))
    else:
        _check(lib.ap_eval_batch_ex(*args, _ptr(n_invalid, "int64", plan.device, 1),
                                    _stream(stream)))


def ap_search_exhaustive(plan: Plan, p: int, m: int, k_lo: int, k_hi: int, rank_lo: int,
                         rank_hi: int, key, stream=None):
    """key: int64 CUDA tensor [1] (written, stream-ordered)."""
    _check(lib.ap_search_exhaustive(plan.handle, int(p), int(m), int(k_lo), int(k_hi),
                                    int(rank_lo), int(rank_hi), _ptr(key, "int64", plan.device),
                                    _stream(stream)))


AP_SEARCH_FULL, AP_SEARCH_KFACTOR, AP_SEARCH_PRUNED, AP_SEARCH_MEMORY = 0, 1, 2, 4


def ap_search_exhaustive_mode(plan: Plan, p: int, m: int, k_lo: int, k_hi: int, rank_lo: int,
                              rank_hi: int, mode: int, key, stream=None):
    """Same key as ap_search_exhaustive; mode selects full / k-factored / pruned."""
    _check(lib.ap_search_exhaustive_mode(plan.handle, int(p), int(m), int(k_lo), int(k_hi),
                                         int(rank_lo), int(rank_hi), int(mode),
                                         _ptr(key, "int64", plan.device), _stream(stream)))


def ap_search_exhaustive2(plan: Plan, p: int, m: int, k_lo: int, k_hi: int, rank_lo: int,
                          rank_hi: int, mode: int, out, stream=None):
    """Two-word reduction: out (device int64[2]) = (least T, least index with it)."""
    _check(lib.ap_search_exhaustive2(plan.handle, int(p), int(m), int(k_lo), int(k_hi),
                                     int(rank_lo), int(rank_hi), int(mode),
                                     _ptr(out, "int64", plan.device, 2), _stream(stream)))


def ap_search_exhaustive_bounded(plan: Plan, p: int, m: int, k_lo: int, k_hi: int, rank_lo: int,
                                 rank_hi: int, mode: int, t_bound: int, out, stream=None):
    """ap_search_exhaustive2 keeping only T <= min(T_ref, t_bound) (t_bound attained)."""
    _check(lib.ap_search_exhaustive_bounded(plan.handle, int(p), int(m), int(k_lo), int(k_hi),
                                            int(rank_lo), int(rank_hi), int(mode), int(t_bound),
                                            _ptr(out, "int64", plan.device, 2), _stream(stream)))


def ap_key2_select(local, t_star, idx, stream=None):
    """idx = local[1] if local[0] == t_star else INT64_MAX (device, stream-ordered)."""
    dev = local.device.index
    _check(lib.ap_key2_select(_ptr(local, "int64", dev, 2), _ptr(t_star, "int64", dev),
                              _ptr(idx, "int64", dev), _stream(stream)))


def ap_search_heuristic(plan: Plan, p: int, m: int, seed: int, radius: int, r_lo: int,
                        r_hi: int, adjust_mode: int, key, stream=None):
    _check(lib.ap_search_heuristic(plan.handle, int(p), int(m), int(seed), int(radius),
                                   int(r_lo), int(r_hi), int(adjust_mode),
                                   _ptr(key, "int64", plan.device), _stream(stream)))


def ap_search_reachable(plan: Plan, p: int, m: int, seed: int, radius: int, r_lo: int,
                        r_hi: int, vmax: int, key, stream=None):
    """Reachable-set (all-children) restarts; key = min (T << 20 | r) (include/ap.h)."""
    _check(lib.ap_search_reachable(plan.handle, int(p), int(m), int(seed), int(radius),
                                   int(r_lo), int(r_hi), int(vmax),
                                   _ptr(key, "int64", plan.device), _stream(stream)))


def ap_decode_reachable(plan: Plan, p: int, m: int, seed: int, radius: int, vmax: int,
                        key: int) -> dict:
    out = ApResult()
    _check(lib.ap_decode_reachable(plan.handle, int(p), int(m), int(seed), int(radius),
                                   int(vmax), int(key), C.byref(out)))
    return _result(out)


def ap_last_truncated() -> int:
    v = C.c_uint64()
    _check(lib.ap_last_truncated(C.byref(v)))
    return v.value


def _result(r: ApResult) -> dict:
    return {"time_ns": r.time_ns, "rank": r.rank, "restart": r.restart, "k": r.k,
            "master": r.master, "p": r.p, "cuts": [int(c) for c in r.cuts[: max(r.p - 1, 0)]]}


def ap_decode(plan: Plan, mode: int, p: int, m: int, k_lo: int = 1, k_hi: int = 1,
              seed: int = 0, radius: int = 0, adjust_mode: int = 0, key: int = 0) -> dict:
    out = ApResult()
    _check(lib.ap_decode(plan.handle, int(mode), int(p), int(m), int(k_lo), int(k_hi), int(seed),
                         int(radius), int(adjust_mode), int(key), C.byref(out)))
    return _result(out)


def ap_slice_sweep(plan: Plan, p: int, m: int, cuts: Sequence[int], k_max: int):
    c = _i32(cuts) if p > 1 else np.zeros(1, np.int32)
    T = np.zeros(int(k_max), np.int64)
    bk = C.c_int32()
    _check(lib.ap_slice_sweep(plan.handle, int(p), int(m), c.ctypes.data_as(C.POINTER(C.c_int32)),
                              int(k_max), T.ctypes.data_as(C.POINTER(C.c_int64)), C.byref(bk)))
    return T, bk.value


def ap_slice_sweep_paper(plan: Plan, p: int, m: int, cuts: Sequence[int], k: int, s_max: int):
    """T(s) for s = 0..s_max with the first s micro-batches' forwards in k pieces."""
    c = _i32(cuts) if p > 1 else np.zeros(1, np.int32)
    T = np.zeros(int(s_max) + 1, np.int64)
    bs = C.c_int32()
    _check(lib.ap_slice_sweep_paper(plan.handle, int(p), int(m),
                                    c.ctypes.data_as(C.POINTER(C.c_int32)), int(k), int(s_max),
                                    T.ctypes.data_as(C.POINTER(C.c_int64)), C.byref(bs)))
    return T, bs.value


def ap_slicer_alg2(plan: Plan, p: int, cuts: Sequence[int], reading: int = 1) -> int:
    """Algorithm 2's mb (reading 0: pseudocode stop test, 1: the text's)."""
    c = _i32(cuts) if p > 1 else np.zeros(1, np.int32)
    mb = C.c_int32()
    _check(lib.ap_slicer_alg2(plan.handle, int(p), c.ctypes.data_as(C.POINTER(C.c_int32)),
                              int(reading), C.byref(mb)))
    return mb.value


def ap_critical_path(plan: Plan, p: int, m: int, k: int, cuts: Sequence[int],
                     cap: Optional[int] = None) -> dict:
    c = _i32(cuts) if p > 1 else np.zeros(1, np.int32)
    cap = cap if cap is not None else p * (2 * m + k)
    ops = (ApOp * max(cap, 1))()
    ln = C.c_int32(); ms = C.c_int32(); T = C.c_int64()
    _check(lib.ap_critical_path(plan.handle, int(p), int(m), int(k),
                                c.ctypes.data_as(C.POINTER(C.c_int32)), ops, int(cap),
                                C.byref(ln), C.byref(ms), C.byref(T)))
    return {"T": T.value, "master": ms.value, "path_len": ln.value,
            "path": [(o.stage, o.kind, o.microbatch, o.piece, o.start_ns, o.end_ns)
                     for o in ops[: ln.value]]}


def ap_alg1(plan: Plan, p: int):
    cuts = np.zeros(AP_MAX_P, np.int32)
    v = C.c_int64()
    _check(lib.ap_alg1(plan.handle, int(p), cuts.ctypes.data_as(C.POINTER(C.c_int32)),
                       C.byref(v)))
    return cuts[: p - 1].copy(), v.value


def ap_plan_set_memory(plan: Plan, static_bytes, stash_bytes, cap_bytes: int):
    """Attach the N4 memory model (include/ap.h) for AP_SEARCH_MEMORY searches."""
    sb = np.ascontiguousarray(static_bytes, dtype=np.int64)
    tb = np.ascontiguousarray(stash_bytes, dtype=np.int64)
    if sb.shape != (plan.n,) or tb.shape != (plan.n,):
        raise ValueError("memory tables must have n entries")
    _check(lib.ap_plan_set_memory(plan.handle, sb.ctypes.data_as(C.POINTER(C.c_int64)),
                                  tb.ctypes.data_as(C.POINTER(C.c_int64)), int(cap_bytes)))


def ap_min_lower_bound(plan: Plan, p: int, m: int, K: int = 1):
    """Certified lower bound on T* over all partitions and k <= K (include/ap.h).
    Returns (lb, cuts of a partition attaining the relaxed bound)."""
    cuts = np.zeros(AP_MAX_P, np.int32)
    v = C.c_int64()
    _check(lib.ap_min_lower_bound(plan.handle, int(p), int(m), int(K), C.byref(v),
                                  cuts.ctypes.data_as(C.POINTER(C.c_int32))))
    return v.value, cuts[: p - 1].copy()


def ap_last_launch() -> dict:
    info = ApLaunchInfo()
    lib.ap_last_launch(C.byref(info))
    return {f: getattr(info, f) for f, _ in ApLaunchInfo._fields_}


def ap_last_kernel_ms() -> float:
    """Device time of the last search's dominant kernel (library CUDA events on the
    caller's stream); the stream must have passed it."""
    v = C.c_float()
    _check(lib.ap_last_kernel_ms(C.byref(v)))
    return float(v.value)


def ap_last_sims() -> int:
    """Simulations run by the last search call on this thread."""
    v = C.c_uint64()
    _check(lib.ap_last_sims(C.byref(v)))
    return int(v.value)


def ap_kernel_launches() -> int:
    """Kernels launched by libap.so since it was loaded (include/ap.h)."""
    return int(lib.ap_kernel_launches())
