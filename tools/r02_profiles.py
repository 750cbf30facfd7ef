"""Write the round-2 profile summaries from a tools/r02_capture.sh run (gpurun_out/)."""
import collections, csv, json, os, shutil, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G = os.path.join(ROOT, "gpurun_out")
P = os.path.join(ROOT, "profiles")


def last_json(path):
    for line in reversed(open(path).read().strip().splitlines()):
        if line.startswith("{"):
            return line
    raise SystemExit(f"no JSON line in {path}")


bl = last_json(os.path.join(G, "r02_bench.json"))
b = json.loads(bl)
open(os.path.join(P, "r02_bench.json"), "w").write(bl + "\n")
open(os.path.join(P, "r02_bench_2rank_gloo_one_gpu.json"), "w").write(
    last_json(os.path.join(G, "r02_bench_2rank_gloo.json")) + "\n")
open(os.path.join(P, "r02_bench_reference.json"), "w").write(
    last_json(os.path.join(G, "r02_bench_reference.json")) + "\n")
shutil.copy(os.path.join(G, "r02_launches.csv"), os.path.join(P, "r02_launches.csv"))
shutil.copy(os.path.join(G, "ncu_sweep_c4.json"), os.path.join(P, "ncu_sweep_c4.json"))
tests = open(os.path.join(G, "r02_pytest.log")).read().strip().splitlines()[-1]
r = b["roofline"]
c5 = b["secondary"]["C5"]
ev = b["secondary"]["eval_batch"]


def txt(name):
    return open(os.path.join(G, name)).read().strip()


open(os.path.join(P, "r02_ncu_sweep.md"), "w").write(f"""# r02 -- ncu `--set full` of the dominant kernel `k_sweep_exact<8, u32, FULL>` (C4)

Command (one B200, `tools/r02_capture.sh` under gpurun):
`ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_sweep_exact<.int.8, unsigned int, .bool.0>" -s 2 -c 1 -o gpurun_out/sweep_c4_r2 python bench.py --steps 1 --warmup 3 --no-secondary --no-cpu-baseline`,
summarised on the box with `tools/ncu_summary.py <report> 5569524480 12 --json profiles/ncu_sweep_c4.json`
(the `.ncu-rep` is too large to bring back; `ncu_sweep_c4.json` is what bench.py attaches as `roofline.ncu` / `roofline.traffic`).

Workload: C4 = n 66, p 8, m 64, k 1..8: 696 190 560 partitions x 8 = 5 569 524 480 simulations in ONE launch
(148 SMs x 3 CTAs x 256 threads, persistent, warp-dynamic work units).  GPU tests on the same build: {tests}.

## Headline (bench.py, same build: `profiles/r02_bench.json`)

| quantity | value |
|---|---|
| kernel time in bench.py (library CUDA events on the launching stream, 10 steps) | {r['kernel_ms_avg']:.2f} ms |
| kernel share of the time-to-plan step | {100*r['kernel_share_of_step']:.2f} % |
| algorithmic int32 ops per launch (DESIGN §5.3: adds + distinct maxima) | {r['ops_per_launch']:.4e} |
| achieved | {r['achieved']:.2f} Tops/s |
| peak (measured 1:1 VIADDMNMX:IMAD, 185.7 int32 ops/clk/SM x 148 x {b['clocks']['sm_mhz']:.0f} MHz; `r02_intpeak.json`) | {r['peak']:.2f} Tops/s |
| **frac** | **{r['frac']:.3f}** (SURVEY §8d naive count: {r['frac_naive_count']:.3f}) |
| DRAM bytes per launch (ncu) | {r['traffic']} B (algorithmic: 0 B per candidate) |
| SM clock during the bench (nvidia-smi, median under load) | {b['clocks']['sm_mhz']} MHz, throttle reasons {b['clocks']['reasons']} |
| candidates/s (whole step) | {b['value']:.4e}; e2e (host tables, copies in the timed region) {b['e2e']['value']:.4e} |

## Raw metrics, stalls, hottest blocks

```
{txt('r02_ncu_sweep.txt')}
```

Executed opcodes (whole kernel, warp-instructions):
```
{txt('sweep_c4_r2.opcodes.txt')}
```

Reading it:
* {txt('r02_ncu_sweep.txt').split('instr/sim ')[1].split()[0]} instructions per simulation; the ALU-pipe ones are VIADDMNMX (467 per
  simulation), VIMNMX (36: warm-up and last slice piece, max-then-add), ISETP/VIADD/LOP3/IADD3
  loop control and successor (~50).  The floor is the 494 distinct maxima per simulation
  (DESIGN §5.3); the ALU pipe is {r['ncu']['alu_pipe_pct']:.0f} % busy.
* The steady loop (the block executed 6 times per simulation, 6 trips x 8 rows) is 7
  VIADDMNMX + 1 IMAD per row, ~45 % of the instructions; the fused cool-down is one
  VIADDMNMX per op.
* Stalls are math_pipe_throttle / not_selected: the pipes, not latency.  No local memory
  in the loops (the class-A codegen of `r02_build_seed.md` keeps 104 B of stack outside them).
""")

open(os.path.join(P, "r02_ncu_heur.md"), "w").write(f"""# r02 -- ncu `--set full` of the heuristic restart kernel `k_heur_pool<16>` (C5)

Command: `ncu --set full --clock-control none --import-source on -k regex:k_heur_pool -s 0 -c 1 -o gpurun_out/heurpool_c5_r2 python tools/c5_once.py 1`
(`tools/r02_capture.sh`).  65 536 restarts, 1 289 183 simulations (p 16, m 64, u32 fast path; the
exact redo pass had 0 restarts).  Bench (same build): C5 time to plan {c5['time_to_plan_ms']:.2f} ms,
{c5['sims_per_s']:.3e} sims/s; the oracle on the same host: {c5['cpu_baseline']['value']:.4g} sims/s.

```
{txt('r02_ncu_heur.txt')}
```

Executed opcodes:
```
{txt('heurpool_c5_r2.opcodes.txt')}
```

Reading it (instr/sim is warp-instructions x 32 / simulations, so idle lanes count):
* The steady rows run as aligned 8-row chunks (the 506-instruction block: 120 decisions,
  per decision one fused add+max, one add, one compare and one predicated IMAD into the
  stage's column word), 5 per simulation, plus the single rows before the first aligned
  row.  Per-sim execution counts above 5 (chunk) and 1 (cool-down, warm-up + weights) are
  lanes a pass leaves idle or gives to speculation (DESIGN §5.6): ~1.3x at 32 slots per
  warp (r02 before this session: ~2x).
* The critical-path walk is one find-last-set per stage change on column words.
* The block at the kernel's end is the CTA's final barrier (warps that are done wait for
  the CTA's last walk).
* C5's walks are bimodal (80 % end within 8 steps, 20 % take 21-29), and the kernel is as
  long as ~30 dependent passes (`r02_heur_pool_variants.md`).
""")

open(os.path.join(P, "r02_ncu_evalfast.md"), "w").write(f"""# r02 -- ncu `--set full` of `k_eval_fast<8>` with the master stage (C4, `ap_eval_batch`)

Command: `ncu --set full --clock-control none --import-source on -k regex:k_eval_fast -s 8 -c 1 -o gpurun_out/evalfast_master_c4_r2 python tools/eval_time.py 4 20`
(the 9th launch is the first T + master call: 2^20 random C4 partitions, k = 1).
Bench (same build, 2^22 partitions, CUDA events): T only {ev['T']['sims_per_s']:.3e} sims/s,
T + master {ev['T_master_k1']['sims_per_s']:.3e} sims/s (round 1: 9.5e9 / 1.98e9).

```
{txt('r02_ncu_evalfast.txt')}
```

Executed opcodes:
```
{txt('evalfast_master_c4_r2.opcodes.txt')}
```
""")

# launch list summary
rows = list(csv.reader(open(os.path.join(G, "r02_launches.csv"))))
hdr = None
agg = collections.OrderedDict()
for rr in rows:
    if "Kernel Name" in rr:
        hdr = {k: i for i, k in enumerate(rr)}
        continue
    if not hdr or len(rr) < len(hdr) or rr[hdr["Metric Name"]] != "gpu__time_duration.sum":
        continue
    name = rr[hdr["Kernel Name"]]
    v = float(rr[hdr["Metric Value"]].replace(",", ""))
    unit = rr[hdr["Metric Unit"]]
    ms = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}[unit] * v
    n, t = agg.get(name, (0, 0.0))
    agg[name] = (n + 1, t + ms)
tot = sum(t for _, t in agg.values())
lines = ["| kernel | launches | total ms | share |", "|---|---|---|---|"]
for name, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    lines.append(f"| `{name[:110]}` | {n} | {t:.3f} | {100*t/tot:.3f}% |")
open(os.path.join(P, "r02_launches_summary.md"), "w").write(f"""# r02 launch list (ncu --metrics gpu__time_duration.sum --clock-control none)

Command: `ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline`
(C4 timed steps, warm-up, e2e steps, the KFACTOR/PRUNED mode runs and every secondary config).
Raw list: `r02_launches.csv`.  Per-launch times are cold-cache and serialised; compare shares, not
absolutes.  The bench's live CUDA-event share of the sweep is {r['kernel_share_of_step']:.3f} of the C4 step.

""" + "\n".join(lines) + "\n")
print("wrote profiles for", b["value"], "sims/s")
