"""CPU oracle timing on the host's cores for all five configs (SURVEY §8(d) "Oracle
timing"): C1/C2 full exhaustive, C3/C4 time-boxed contiguous samples at evenly spaced
ranks (rate + extrapolated full time, labelled), C5 a restart sample of the heuristic.
The oracle runs as it stands (plain C behind ctypes, one thread per core).  Writes a
markdown table to stdout.  usage: oracle_timing.py [seconds_per_sample]"""
import os
import sys
import time
from concurrent.futures import ThreadPoolExecutor
from math import comb

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402  (test infrastructure; this tool only reports its speed)
import synth  # noqa: E402

budget = float(sys.argv[1]) if len(sys.argv) > 1 else 5.0
threads = os.cpu_count() or 1


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


rows = []
for cfg in (1, 2, 3, 4):
    wl = synth.config(cfg)
    M = oracle.Model.from_workload(wl)
    N = comb(wl.n - 1, wl.p - 1)
    K = wl.k_hi - wl.k_lo + 1
    if cfg <= 2:
        t0 = time.perf_counter()
        o = M.exhaustive_parallel(wl.p, wl.m, wl.k_lo, wl.k_hi, threads=threads)
        dt = time.perf_counter() - t0
        rows.append((wl.name, "full exhaustive", N * K, dt, N * K / dt, dt, o["T"]))
        continue
    t0 = time.perf_counter()
    M.exhaustive(wl.p, wl.m, wl.k_lo, wl.k_hi, 0, 64)
    per_sim = (time.perf_counter() - t0) / (64 * K)
    per = max(1, int(budget / per_sim / K / threads))
    starts = [int(N * i / threads) for i in range(threads)]
    t0 = time.perf_counter()
    with ThreadPoolExecutor(threads) as ex:
        res = list(ex.map(lambda s: M.exhaustive(wl.p, wl.m, wl.k_lo, wl.k_hi, s, min(N, s + per)),
                          starts))
    dt = time.perf_counter() - t0
    sims = sum(r["sims"] for r in res)
    rate = sims / dt
    rows.append((wl.name, f"sample: {threads} windows x {per} partitions x {K} k", sims, dt, rate,
                 N * K / rate, None))
wl = synth.config(5)
M = oracle.Model.from_workload(wl)
R = 4096
t0 = time.perf_counter()
o = M.heuristic_parallel(wl.p, wl.m, wl.seed, wl.radius, 0, R, threads=threads)
dt = time.perf_counter() - t0
rows.append((wl.name, f"heuristic: restarts [0, {R})", o["sims"], dt, o["sims"] / dt,
             dt * wl.restarts / R, o["T"]))

print(f"Host: {threads} threads, {cpu_model()}\n")
print("| config | what was timed | simulations | wall s | sims/s | full job s (extrapolated where sampled) | T found |")
print("|---|---|---|---|---|---|---|")
for name, what, sims, dt, rate, full, T in rows:
    print(f"| {name} | {what} | {sims} | {dt:.2f} | {rate:.3e} | {full:.1f} | {T if T is not None else '-'} |")
