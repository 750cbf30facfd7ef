#!/usr/bin/env python
"""Bench: candidate schedules simulated/s and time-to-optimal-plan (BASELINE.json).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 4] [--impl ours|reference]

One step = one pass of the whole hot path over the
workload: Algorithm 1 + T_ref, the exhaustive sweep of this rank's shard of all
C(n-1,p-1) partitions x k (every pair fully simulated), the per-GPU argmin, ONE NCCL
all_reduce(MIN) of the packed 8-byte key (N>1), decode (unrank + critical path +
master stage) and the Slicer sweep of the winner.  Default workload = BASELINE.json
configs[3] (C4, GPT-3-2.7B-shaped, n=66, p=8, m=64, k in 1..8: 5.57e9 simulations),
the largest exhaustive config.  Multi-GPU: the rank space is split across ranks
("strong" scaling: total work fixed); value = all simulations / max-over-ranks time.

Rank 0 prints ONE JSON line.  See DESIGN.md §7 for every field.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402

METRIC = "candidate schedules simulated/sec"
MEASURED = os.path.join(ROOT, "MEASURED_PEAKS.json")


def _env_rank():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("LOCAL_RANK", 0)),
            int(os.environ.get("WORLD_SIZE", 1)))


def _peaks():
    try:
        with open(MEASURED) as fh:
            d = json.load(fh)
        return d, "measured"
    except Exception:
        return {"sm_max_mhz": 1965.0}, "fallback"


INTPEAK = os.path.join(ROOT, "profiles", "r02_intpeak.json")


def int_peak(sm_mhz: float, sms: int = 148):
    """Integer roofline in int32 ops/s.  The max-plus work runs on two
    pipes: the ALU pipe, whose VIADDMNMX does two int32 ops (add + max), and the FMA pipe,
    whose IMAD does one add.  The denominator is MEASURED on the B200 by the builder's
    microbenchmark (tools/microbench/intpeak.cu, committed result profiles/r02_intpeak.json):
    a 1:1 VIADDMNMX:IMAD mix with 8 independent chains per thread reaches 185.7 int32
    ops/clk/SM (0.967 warp-instructions/clk/SMSP; the two single-pipe rates are 0.499
    each).  Scaled to the clock measured during the bench's timed region.
    Returns (ops/s, ops/clk/SM, source string)."""
    try:
        with open(INTPEAK) as fh:
            d = json.load(fh)
        per = float(d["modes"]["mix11"]["int32_ops_per_clk_per_sm"])
        src = ("measured (builder microbench tools/microbench/intpeak.cu, 1:1 VIADDMNMX:IMAD, "
               f"profiles/r02_intpeak.json: {per:.1f} int32 ops/clk/SM)")
    except Exception:
        per = 192.0
        src = "fallback: 64 ALU lanes x 2 ops + 64 FMA lanes x 1 op per clk per SM (guide pipe rates)"
    return sms * per * sm_mhz * 1e6, per, src


NCU_PROFILE = os.path.join(ROOT, "profiles", "ncu_sweep_c4.json")


def _ncu_profile():
    """Per-launch figures of the dominant kernel from the committed ncu --set full
    capture (tools/ncu_summary.py --json writes it): DRAM bytes, issue/pipe use."""
    try:
        with open(NCU_PROFILE) as fh:
            return json.load(fh)
    except Exception:
        return None


def ops_per_sim(p: int, m: int, k: int) -> int:
    """Algorithmic int32 ops of one simulation: one add per op of
    the task DAG (its weight, receive comm included) plus one max per DISTINCT pair
    of predecessors.  B(x,y) and F(x+1, y+w_x) have the same two predecessors
    (B(x+1,y), F(x,y+w_x)) wherever w_x = w_{x+1}+1, so that max is counted once.
    The naive count of SURVEY.md §8d (2 ops per op) is ops_per_sim_naive."""
    nops = p * (2 * m + k - 1)
    w = [min(p - 1 - x, m) for x in range(p)]
    two_pred = (p - 1) * (m - 1 + k - 1) + (p - 1) * m
    shared = sum(m - w[x] for x in range(p - 1) if w[x] == w[x + 1] + 1)
    return nops + two_pred - shared


def ops_per_sim_naive(p: int, m: int, k: int) -> int:
    """2pm + (k-1)p max-plus ops, one max + one add each."""
    return 2 * (2 * p * m + (k - 1) * p)


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled DURING the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap,power.draw")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self._t = threading.Thread(target=self._read, daemon=True)
            self._t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0])); smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "samples": len(sm), "reasons": sorted(reasons)}


def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


# ----------------------------------------------------------------------------- oracle
def _oracle_window_rate(M, wl, N, budget_s, threads, nwin):
    """One time-boxed oracle run: `nwin` contiguous lex-rank windows starting at evenly
    spaced ranks; `threads` host threads visit their windows round-robin, simulating one
    batch of ~256 (partition, k) pairs per visit (the C oracle releases the GIL), until
    `budget_s` of wall time has passed.  Each thread calibrates itself: it stops on its own
    clock, so a slow core does not hold the others."""
    from concurrent.futures import ThreadPoolExecutor
    K = wl.k_hi - wl.k_lo + 1
    batch = max(1, 256 // K)
    starts = [N * i // nwin for i in range(nwin)]
    pos = list(starts)
    ends = [starts[i + 1] if i + 1 < nwin else N for i in range(nwin)]
    t0 = time.perf_counter()

    def worker(t):
        sims = 0
        mine = list(range(t, nwin, threads))
        while time.perf_counter() - t0 < budget_s:
            progressed = False
            for w in mine:
                if pos[w] >= ends[w]:
                    continue
                hi = min(ends[w], pos[w] + batch)
                sims += M.exhaustive(wl.p, wl.m, wl.k_lo, wl.k_hi, pos[w], hi)["sims"]
                pos[w] = hi
                progressed = True
                if time.perf_counter() - t0 >= budget_s:
                    break
            if not progressed:
                break
        return sims

    with ThreadPoolExecutor(threads) as ex:
        per = list(ex.map(worker, range(threads)))
    dt = time.perf_counter() - t0
    return sum(per), dt


def oracle_rate(wl, budget_s: float = 10.0, runs: int = 3, threads: int = 0):
    """The oracle as it stands (plain C DAG simulator, brute force in lex order) on the
    host's cores, on a bounded sample of the workload: `runs` time-boxed
    runs of `budget_s` each over max(8, threads) evenly spaced contiguous rank windows,
    all k; the median rate is reported with the spread of the runs."""
    import oracle
    M = oracle.Model.from_workload(wl)
    N = oracle.count(wl.n, wl.p)
    threads = threads or os.cpu_count() or 1
    nwin = max(8, threads)
    rates, sims_tot, wall_tot = [], 0, 0.0
    for _ in range(runs):
        sims, dt = _oracle_window_rate(M, wl, N, budget_s, threads, nwin)
        rates.append(sims / dt)
        sims_tot += sims
        wall_tot += dt
    med = statistics.median(rates)
    return {"value": med, "unit": "sims/s", "cores": threads, "kind": "oracle",
            "sims": sims_tot, "wall_s": wall_tot,
            "runs": [round(r, 1) for r in rates],
            "spread": (max(rates) - min(rates)) / med if med > 0 else None,
            "sample": f"median of {runs} runs of {budget_s:.0f} s wall, each over {nwin} "
                      f"contiguous lex-rank windows at evenly spaced start ranks of the "
                      f"{N}-partition space, k in [{wl.k_lo},{wl.k_hi}], {threads} host threads "
                      f"time-boxed on their own clocks ({sims_tot} simulations in {wall_tot:.1f} s)",
            "cpu": cpu_model()}


def oracle_full_exhaustive(wl, runs: int = 3, threads: int = 0):
    """The oracle's COMPLETE exhaustive search of a small config (C1, C2: BASELINE.md §4
    'full exhaustive run, timed') on the host's cores: time to its optimal plan and
    simulations/s, median of `runs`; its argmin is returned for comparison."""
    import oracle
    M = oracle.Model.from_workload(wl)
    threads = threads or os.cpu_count() or 1
    ts, o = [], None
    for _ in range(runs):
        t0 = time.perf_counter()
        o = M.exhaustive_parallel(wl.p, wl.m, wl.k_lo, wl.k_hi, threads=threads)
        ts.append(time.perf_counter() - t0)
    med = statistics.median(ts)
    return {"value": o["sims"] / med, "unit": "sims/s", "cores": threads, "kind": "oracle",
            "time_to_optimal_plan_ms": 1e3 * med, "runs_ms": [round(1e3 * t, 2) for t in ts],
            "T_ns": o["T"], "rank": o["rank"], "k": o["k"],
            "sample": f"the whole search ({o['sims']} simulations), median of {runs} runs, "
                      f"{threads} host threads", "cpu": cpu_model()}


def oracle_heuristic_rate(wl, restarts: int = 4096, runs: int = 3, threads: int = 0):
    """The oracle's heuristic (O9) over a fixed sample of restarts [0, restarts) on the
    host's cores: simulations/s and restarts/s, median of `runs`."""
    import oracle
    M = oracle.Model.from_workload(wl)
    threads = threads or os.cpu_count() or 1
    rates = []
    for _ in range(runs):
        t0 = time.perf_counter()
        o = M.heuristic_parallel(wl.p, wl.m, wl.seed, wl.radius, 0, restarts, threads=threads)
        dt = time.perf_counter() - t0
        rates.append((o["sims"] / dt, restarts / dt))
    med = statistics.median(r[0] for r in rates)
    return {"value": med, "unit": "sims/s", "cores": threads, "kind": "oracle",
            "restarts_per_s": statistics.median(r[1] for r in rates),
            "runs": [round(r[0], 1) for r in rates],
            "spread": (max(r[0] for r in rates) - min(r[0] for r in rates)) / med,
            "sample": f"restarts [0, {restarts}) of the {wl.restarts}-restart search, "
                      f"median of {runs} runs, {threads} host threads", "cpu": cpu_model()}


def run_reference(args):
    rank, local, world = _env_rank()
    if rank != 0:
        return 0
    wl = synth.config(args.config)
    steps = []
    for i in range(args.warmup + args.steps):
        r = oracle_rate(wl, budget_s=args.ref_budget, runs=1)
        if i >= args.warmup:
            steps.append(r)
    val = statistics.median(r["value"] for r in steps)
    cb = dict(steps[-1])
    cb["value"] = val
    cb["runs"] = [round(r["value"], 1) for r in steps]
    cb["spread"] = (max(cb["runs"]) - min(cb["runs"])) / val if val > 0 else None
    cb["sample"] = (f"{args.steps} timed steps (after {args.warmup} warm-up), each one "
                    f"time-boxed run: " + steps[-1]["sample"].split(", each over ", 1)[-1])
    N = synth_count(wl)
    total = N * (wl.k_hi - wl.k_lo + 1)
    out = {"impl": "reference", "metric": METRIC, "value": val, "unit": "sims/s",
           "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
           "ms_per_step": 1e3 * statistics.median(r["wall_s"] for r in steps),
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
           "dtype": "int64", "data": "synthetic",
           "config": {"workload": wl.name, "n": wl.n, "p": wl.p, "m": wl.m,
                      "k": [wl.k_lo, wl.k_hi], "search": wl.search, "total_sims": total,
                      "extrapolated_time_to_plan_s": total / val},
           "cpu_baseline": cb,
           "e2e": {"value": val, "unit": "sims/s", "h2d_bytes_per_step": 0,
                   "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


def synth_count(wl):
    from math import comb
    return comb(wl.n - 1, wl.p - 1)


# ----------------------------------------------------------------------------- ours
def main():
    ap_ = argparse.ArgumentParser()
    ap_.add_argument("--gpus", type=int, default=1)
    ap_.add_argument("--steps", type=int, default=10)
    ap_.add_argument("--warmup", type=int, default=3)
    ap_.add_argument("--config", type=int, default=4)
    ap_.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap_.add_argument("--no-cpu-baseline", action="store_true")
    ap_.add_argument("--no-secondary", action="store_true")
    ap_.add_argument("--ref-budget", type=float, default=8.0)
    ap_.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                     help="process-group backend (gloo + --device-override only to "
                          "exercise the sharded path on a one-GPU box)")
    ap_.add_argument("--device-override", type=int, default=None)
    args = ap_.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    import paper_conf_cluster_liulldgl22_b200 as ap
    from paper_conf_cluster_liulldgl22_b200.search import shard

    rank, local, world = _env_rank()
    if args.device_override is not None:
        local = args.device_override
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if args.backend == "nccl":
            # communicator-init logging stays on (stderr), so a scaling run shows every
            # rank joining the NCCL communicator
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
        print(f"[bench] rank {rank}/{world} backend {args.backend} on cuda:{local}",
              file=sys.stderr, flush=True)
    peaks, peak_src = _peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    sms = torch.cuda.get_device_properties(local).multi_processor_count

    wl = synth.config(args.config)
    f, b, a = wl.arrays()
    K = wl.k_hi - wl.k_lo + 1
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=local)
    N = ap.ap_count(wl.n, wl.p)
    lo, hi = shard(N, rank, world)
    total_sims = N * K
    my_ops = (hi - lo) * sum(ops_per_sim(wl.p, wl.m, k) for k in range(wl.k_lo, wl.k_hi + 1))
    my_ops_naive = (hi - lo) * sum(ops_per_sim_naive(wl.p, wl.m, k)
                                   for k in range(wl.k_lo, wl.k_hi + 1))
    key = torch.empty(1, dtype=torch.int64, device=dev)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)  # > 126 MB L2

    def step(pl):
        """One time-to-optimal-plan pass through the public C-ABI binding."""
        if hi > lo:
            ap.ap_search_exhaustive(pl, wl.p, wl.m, wl.k_lo, wl.k_hi, lo, hi, key)
        else:
            key.fill_(ap.INT64_MAX)
        if world > 1:
            dist.all_reduce(key, op=dist.ReduceOp.MIN)
        kv = int(key.item())
        res = ap.ap_decode(pl, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=kv)
        Tk, bk = ap.ap_slice_sweep(pl, wl.p, wl.m, res["cuts"], wl.k_hi)
        return res, Tk, bk

    for _ in range(args.warmup):
        res, Tk, bk = step(plan)
    # ------------------------------------------------------------- timed region
    gpu_idx = local
    cvd = os.environ.get("CUDA_VISIBLE_DEVICES")
    if cvd:
        try:
            gpu_idx = int(cvd.split(",")[local])
        except ValueError:
            pass
    clocks = ClockSampler(gpu_idx)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    kern_ms = []
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    time.sleep(0.3)
    launches0 = ap.ap_kernel_launches()
    wall0 = time.perf_counter()
    for i in range(args.steps):
        flush.zero_()                      # L2 flush between timed steps (untimed)
        ev[i][0].record()
        res, Tk, bk = step(plan)
        ev[i][1].record()
        torch.cuda.synchronize()
        if hi > lo:
            kern_ms.append(ap.ap_last_kernel_ms())
    torch.cuda.synchronize()
    launches = ap.ap_kernel_launches() - launches0
    if world > 1:
        dist.barrier()
    wall = time.perf_counter() - wall0
    clk = clocks.stop()
    step_ms = [s.elapsed_time(e) for s, e in ev]
    t_local = sum(step_ms) / 1e3
    tt = torch.tensor([t_local, sum(kern_ms) / 1e3 if kern_ms else 0.0], dtype=torch.float64,
                      device=dev)
    if world > 1:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    t_max, kern_max = float(tt[0]), float(tt[1])
    value = total_sims * args.steps / t_max
    info = ap.ap_last_launch()

    # ------------------------------------------------------------- e2e (host buffers)
    e2e_steps = max(3, min(args.steps, 5))
    tab_bytes = 3 * ((wl.n + 1) & ~1) * 8 + (wl.n + 1) * 33 * 8
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        pl = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=local)   # H2D tables
        step(pl)                                                            # D2H key/result
        pl.close()
    torch.cuda.synchronize()
    e2e_t = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    e2e_val = total_sims * e2e_steps / float(e2e_t[0])

    # ------------------------------------------------------------- other search modes
    # Same exact key, less work per candidate: labelled
    # time-to-optimal-plan numbers, NOT the candidates/s headline (which is defined on
    # the full per-(partition, k) sweep above).
    modes = {}
    for mode, name in ((ap.AP_SEARCH_KFACTOR, "kfactor"), (ap.AP_SEARCH_PRUNED, "pruned")):
        kk = torch.empty(1, dtype=torch.int64, device=dev)
        def run_mode():
            """The same time-to-optimal-plan path as step(): search, reduction, decode
            (unrank + critical path + master) and the Slicer sweep of the winner."""
            if hi > lo:
                ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, lo, hi, mode, kk)
            else:
                kk.fill_(ap.INT64_MAX)
            if world > 1:
                dist.all_reduce(kk, op=dist.ReduceOp.MIN)
            kv_ = int(kk.item())
            res_ = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=kv_)
            ap.ap_slice_sweep(plan, wl.p, wl.m, res_["cuts"], wl.k_hi)
            return kv_
        for _ in range(3):
            run_mode()
        ts = []
        for _ in range(5):
            flush.zero_()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); kv = run_mode(); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        tmed = torch.tensor([statistics.median(ts)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(tmed, op=dist.ReduceOp.MAX)
        modes[name] = {"time_to_optimal_plan_ms": float(tmed[0]),
                       "path": "search + all_reduce + decode + Slicer sweep (as the step)",
                       "same_key_as_full": kv == int(key.item()),
                       "equivalent_candidates_per_s": total_sims / (float(tmed[0]) / 1e3)}

    # ------------------------------------------------------------- secondary workloads
    secondary = {}
    if not args.no_secondary:
        secondary = run_secondary(ap, torch, dist, world, rank, dev, shard)

    # ------------------------------------------------------------- roofline
    k_avg_s = kern_max / max(len(kern_ms), 1)
    achieved = my_ops / k_avg_s if k_avg_s > 0 else 0.0
    clk_mhz = clk.get("sm_mhz") or sm_max
    peak, per_clk, peak_src = int_peak(clk_mhz, sms)
    # the same roofline for the secondary kernels (achieved algorithmic int32 ops / time)
    def sec_roof(kernel, sims, p_, m_, ks, ms):
        if not ms or ms <= 0:
            return None
        ops = sims * statistics.mean(ops_per_sim(p_, m_, k) for k in ks)
        naive = sims * statistics.mean(ops_per_sim_naive(p_, m_, k) for k in ks)
        a = ops / (ms / 1e3)
        return {"bound": "alu", "kernel": kernel, "achieved": a / 1e12, "peak": peak / 1e12,
                "unit": "Tops/s (int32)", "frac": a / peak,
                "frac_naive_count": naive / (ms / 1e3) / peak, "time_ms": ms}
    if secondary.get("C5"):
        c5 = secondary["C5"]
        c5["roofline"] = sec_roof("k_heur_pool<16> (restart kernel)", c5["sims_per_step"] / max(world, 1),
                                  16, 64, [1], c5.get("kernel_ms"))
    if secondary.get("eval_batch"):
        evb = secondary["eval_batch"]
        w4 = synth.config(4)
        for name, ks in (("T", range(w4.k_lo, w4.k_hi + 1)), ("T_master_k1", [1])):
            if name in evb:
                evb[name]["roofline"] = sec_roof("k_eval_fast<8> (+ exact redo pass)", 1 << 22, w4.p, w4.m,
                                                 list(ks), evb[name]["ms"])
    roof = {"bound": "alu", "kernel": "k_sweep_exact<%d,%s>" % (wl.p, "u32" if info["fast_u32"] else "u64"),
            "achieved": achieved / 1e12, "peak": peak / 1e12, "unit": "Tops/s (int32)",
            "frac": achieved / peak, "traffic": None,
            "count": "adds + distinct maxima of the 1F1B task DAG (DESIGN.md §5.3)",
            "ops_per_launch": my_ops, "ops_per_sim_avg": my_ops / max(hi - lo, 1) / K,
            "frac_naive_count": (my_ops_naive / k_avg_s / peak) if k_avg_s > 0 else None,
            "naive_count": "SURVEY §8d: 2 int32 ops (max + add) per max-plus op, "
                           "2pm + (k-1)p max-plus ops per simulation",
            "ops_per_sim_naive_avg": my_ops_naive / max(hi - lo, 1) / K,
            "kernel_ms_avg": k_avg_s * 1e3,
            "kernel_share_of_step": (kern_max / t_max) if t_max > 0 else None,
            "peak_source": f"{sms} SMs x {per_clk:.1f} int32 ops/clk/SM x {clk_mhz:.0f} MHz "
                           f"(median SM clock in the timed region); {peak_src}",
            "traffic_note": "algorithmic HBM bytes per candidate = 0; traffic = ncu "
                            "dram__bytes_read+write of this kernel, one --set full capture"}
    prof = _ncu_profile()
    if prof:
        roof["traffic"] = prof.get("dram_bytes_per_launch")
        roof["ncu"] = prof
    out = {"metric": METRIC, "value": value, "unit": "sims/s", "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup,
           "ms_per_step": 1e3 * t_max / args.steps,
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
           "dtype": "u32" if info["fast_u32"] else "int64", "data": "synthetic",
           "config": {"workload": wl.name, "n": wl.n, "p": wl.p, "m": wl.m, "k": [wl.k_lo, wl.k_hi],
                      "search": "exhaustive", "sims_per_step": total_sims,
                      "parallelism": f"rank-space shards x{world}",
                      "l2": "flushed between timed steps (256 MiB write); tables are 2.4 KB",
                      "arith": "u32 saturating at T_ref+1, exact for every candidate that can "
                               "win (DESIGN.md §5.2)" if info["fast_u32"] else "int64",
                      "time_to_optimal_plan_ms": 1e3 * t_max / args.steps,
                      "wall_s": wall},
           "result": {"T_ns": res["time_ns"], "rank": res["rank"], "k": res["k"],
                      "cuts": res["cuts"], "master": res["master"], "slicer_best_k": bk},
           "roofline": roof,
           "clocks": clk,
           "gpu_launches": launches,
           "gpu_launches_note": "libap.so kernels launched in the timed region "
                                "(ap_kernel_launches difference), all ranks' own counts equal",
           "e2e": {"value": e2e_val, "unit": "sims/s", "h2d_bytes_per_step": tab_bytes,
                   "d2h_bytes_per_step": 8 + 8 + 140 + 8 * wl.k_hi, "steps": e2e_steps,
                   "path": "ap_plan_create(host tables) -> ap_search_exhaustive -> "
                           "all_reduce -> ap_decode -> ap_slice_sweep -> ap_plan_destroy"},
           "search_modes": modes,
           "secondary": secondary}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        out["cpu_baseline"] = oracle_rate(wl)
        if not args.no_secondary:
            # same-run oracle rates beside the secondary GPU numbers
            for ci in (1, 2):
                cb = oracle_full_exhaustive(synth.config(ci))
                sec = out["secondary"][f"C{ci}"]
                cb["same_plan_as_gpu"] = (cb["T_ns"], cb["rank"], cb["k"]) == \
                    (sec["T_ns"], sec["rank"], sec["k"])
                sec["cpu_baseline"] = cb
            out["secondary"]["C3"]["cpu_baseline"] = oracle_rate(synth.config(3), budget_s=3.0)
            out["secondary"]["C5"]["cpu_baseline"] = oracle_heuristic_rate(synth.config(5))
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def run_secondary(ap, torch, dist, world, rank, dev, shard):
    """C1/C2/C3 exhaustive and C5 heuristic (65 536 restarts + Slicer sweep), fewer steps."""
    out = {}
    # C1, C2: the whole time-to-optimal-plan path (search, all-reduce, decode with critical
    # path, Slicer sweep over the config's k range), median of 20 CUDA-event-timed runs
    for ci in (1, 2):
        wl = synth.config(ci)
        f, b, a = wl.arrays()
        plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=dev.index)
        N = ap.ap_count(wl.n, wl.p)
        lo, hi = shard(N, rank, world)
        key = torch.empty(1, dtype=torch.int64, device=dev)

        def s12():
            if hi > lo:
                ap.ap_search_exhaustive(plan, wl.p, wl.m, wl.k_lo, wl.k_hi, lo, hi, key)
            else:
                key.fill_(2 ** 63 - 1)
            if world > 1:
                dist.all_reduce(key, op=dist.ReduceOp.MIN)
            res = ap.ap_decode(plan, 0, wl.p, wl.m, wl.k_lo, wl.k_hi, key=int(key.item()))
            ap.ap_slice_sweep(plan, wl.p, wl.m, res["cuts"], max(wl.k_hi, 1))
            return res
        for _ in range(3):
            s12()
        times = []
        for _ in range(20):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); r12 = s12(); e1.record(); torch.cuda.synchronize()
            times.append(e0.elapsed_time(e1))
        t = torch.tensor([statistics.median(times)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        sims = N * (wl.k_hi - wl.k_lo + 1)
        out[f"C{ci}"] = {"workload": wl.name, "sims_per_step": sims,
                         "time_to_optimal_plan_ms": float(t[0]),
                         "sims_per_s": sims / (float(t[0]) / 1e3), "T_ns": r12["time_ns"],
                         "rank": r12["rank"], "k": r12["k"], "cuts": r12["cuts"],
                         "master": r12["master"]}
    # C3
    wl = synth.config(3)
    f, b, a = wl.arrays()
    plan = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=dev.index)
    N = ap.ap_count(wl.n, wl.p)
    lo, hi = shard(N, rank, world)
    key = torch.empty(1, dtype=torch.int64, device=dev)

    def s3():
        ap.ap_search_exhaustive(plan, wl.p, wl.m, 1, 1, lo, hi, key)
        if world > 1:
            dist.all_reduce(key, op=dist.ReduceOp.MIN)
        return ap.ap_decode(plan, 0, wl.p, wl.m, 1, 1, key=int(key.item()))
    for _ in range(3):
        s3()
    times = []
    for _ in range(5):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); r3 = s3(); e1.record(); torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1))
    t = torch.tensor([statistics.median(times)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    out["C3"] = {"workload": wl.name, "sims_per_s": N / (float(t[0]) / 1e3),
                 "time_to_optimal_plan_ms": float(t[0]), "T_ns": r3["time_ns"], "cuts": r3["cuts"]}
    # the pruned exact search (same key) captured once in a CUDA graph and replayed: the
    # search is stream-ordered end to end (no host synchronisation inside it)
    try:
        gk = torch.empty(1, dtype=torch.int64, device=dev)
        side = torch.cuda.Stream()
        side.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(side):
            ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, 1, 1, lo, hi, ap.AP_SEARCH_PRUNED, gk)
        torch.cuda.current_stream().wait_stream(side)
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            ap.ap_search_exhaustive_mode(plan, wl.p, wl.m, 1, 1, lo, hi, ap.AP_SEARCH_PRUNED, gk)
        graph.replay()
        torch.cuda.synchronize()
        times = []
        for _ in range(10):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); graph.replay(); e1.record(); torch.cuda.synchronize()
            times.append(e0.elapsed_time(e1))
        if world > 1:
            dist.all_reduce(gk, op=dist.ReduceOp.MIN)
        out["C3"]["pruned_search_graph_replay_ms"] = statistics.median(times)
        out["C3"]["pruned_graph_key_equals_full"] = int(gk.item()) == int(key.item())
    except Exception as e:  # a capture failure is reported, not hidden
        out["C3"]["pruned_search_graph_error"] = repr(e)
    # C5
    wl = synth.config(5)
    f, b, a = wl.arrays()
    plan5 = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=dev.index)
    rlo, rhi = shard(wl.restarts, rank, world)

    k5 = []  # the restart kernel's own CUDA-event time (library events, launching stream)

    def s5():
        ap.ap_search_heuristic(plan5, wl.p, wl.m, wl.seed, wl.radius, rlo, rhi, 0, key)
        if world > 1:
            dist.all_reduce(key, op=dist.ReduceOp.MIN)
        kv = int(key.item())  # the step's one host read of the key (decode needs it)
        k5.append(ap.ap_last_kernel_ms())
        res = ap.ap_decode(plan5, 1, wl.p, wl.m, seed=wl.seed, radius=wl.radius, key=kv)
        Tk, bk = ap.ap_slice_sweep(plan5, wl.p, wl.m, res["cuts"], wl.slice_k_max)
        return res, Tk, bk
    s5()
    times = []
    kt = []
    for _ in range(3):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); r5, Tk, bk = s5(); e1.record(); torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1))
    t = torch.tensor([statistics.median(times)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    sims5 = torch.tensor([float(ap.ap_last_sims())], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(sims5, op=dist.ReduceOp.SUM)
    out["C5"] = {"workload": wl.name, "restarts": wl.restarts,
                 "restarts_per_s": wl.restarts / (float(t[0]) / 1e3),
                 "sims_per_step": int(sims5[0]),
                 "sims_per_s": float(sims5[0]) / (float(t[0]) / 1e3),
                 "time_to_plan_ms": float(t[0]), "T_ns": r5["time_ns"], "restart": r5["restart"],
                 "cuts": r5["cuts"], "slicer_T_ns": [int(x) for x in Tk], "slicer_best_k": bk,
                 "kernel_ms": statistics.median(k5[1:]) if len(k5) > 1 else None}
    # certified bound (NEXT N3): T* >= minLB, so the plan is within `certified_gap` of optimal
    lb, _ = ap.ap_min_lower_bound(plan5, wl.p, wl.m, 1)
    out["C5"]["certified_minlb_ns"] = lb
    out["C5"]["certified_gap"] = (r5["time_ns"] - lb) / lb

    # reachable-set search (NEXT N1) over the same restarts
    vmax = 1024

    def s5r():
        ap.ap_search_reachable(plan5, wl.p, wl.m, wl.seed, wl.radius, rlo, rhi, vmax, key)
        if world > 1:
            dist.all_reduce(key, op=dist.ReduceOp.MIN)
        return ap.ap_decode_reachable(plan5, wl.p, wl.m, wl.seed, wl.radius, vmax, int(key.item()))
    s5r()
    times = []
    for _ in range(3):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); rr = s5r(); e1.record(); torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1))
    t = torch.tensor([statistics.median(times)], dtype=torch.float64, device=dev)
    st = torch.tensor([float(ap.ap_last_sims()), float(ap.ap_last_truncated())],
                      dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(st, op=dist.ReduceOp.SUM)
    out["C5_reachable"] = {"workload": wl.name + "-reachable-set", "restarts": wl.restarts,
                           "vmax": vmax, "time_to_plan_ms": float(t[0]),
                           "sims_per_step": int(st[0]), "truncated_restarts": int(st[1]),
                           "sims_per_s": float(st[0]) / (float(t[0]) / 1e3),
                           "T_ns": rr["time_ns"], "restart": rr["restart"]}

    # outer loop over pipeline depth with the memory model (NEXT N4)
    from paper_conf_cluster_liulldgl22_b200.search import plan_pipeline_depth
    dw = synth.depth_config()
    f, b, a = dw.base.arrays()
    plan4 = ap.ap_plan_create(f, b, a, dw.base.link_bytes_per_s, device=dev.index)
    ap.ap_plan_set_memory(plan4, dw.static_bytes, dw.stash_bytes, dw.cap_bytes)
    plan_pipeline_depth(plan4, dw.n_gpus, dw.microbatches)
    times = []
    for _ in range(3):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); r4 = plan_pipeline_depth(plan4, dw.n_gpus, dw.microbatches); e1.record()
        torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1))
    t = torch.tensor([statistics.median(times)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    out["N4_depth"] = {"workload": dw.name, "time_to_plan_ms": float(t[0]),
                       "sims_per_step": sum(r["sims"] for r in r4["per_depth"]),
                       "best": {k: r4["best"][k] for k in ("p", "dp", "m", "T", "cuts")},
                       "per_depth_T_ns": {r["p"]: r["T"] for r in r4["per_depth"]}}

    # ap_eval_batch on 2^22 random C4 candidates per rank (T with k in 1..8; T + master
    # at k = 1): the general evaluation entry point, candidates resident in HBM
    wl = synth.config(4)
    f, b, a = wl.arrays()
    plan5 = ap.ap_plan_create(f, b, a, wl.link_bytes_per_s, device=dev.index)
    cnt = 1 << 22
    g = torch.Generator(device=dev)
    g.manual_seed(1234 + rank)
    cuts = torch.sort(torch.argsort(torch.rand(cnt, wl.n - 1, device=dev, generator=g), dim=1)
                      [:, : wl.p - 1] + 1, dim=1).values.to(torch.int32).contiguous()
    ks = torch.randint(wl.k_lo, wl.k_hi + 1, (cnt,), device=dev, generator=g, dtype=torch.int32)
    k1 = torch.ones(cnt, dtype=torch.int32, device=dev)
    Tv = torch.empty(cnt, dtype=torch.int64, device=dev)
    Mv = torch.empty(cnt, dtype=torch.int32, device=dev)
    ev = {}
    for name, kk, mm in (("T", ks, None), ("T_master_k1", k1, Mv)):
        ap.ap_eval_batch(plan5, wl.p, wl.m, cuts, kk, Tv, mm)
        times = []
        for _ in range(5):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); ap.ap_eval_batch(plan5, wl.p, wl.m, cuts, kk, Tv, mm); e1.record()
            torch.cuda.synchronize()
            times.append(e0.elapsed_time(e1))
        t = torch.tensor([statistics.median(times)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ev[name] = {"ms": float(t[0]), "sims_per_s": world * cnt / (float(t[0]) / 1e3)}
    del cuts, ks, k1, Tv, Mv
    out["eval_batch"] = {"workload": "C4 random partitions, 2^22 per rank", **ev}
    return out


if __name__ == "__main__":
    sys.exit(main())
