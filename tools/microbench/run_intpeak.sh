#!/bin/bash
# Measure the integer roofline denominator on the GPU box:
# compile intpeak.cu for sm_100a, run it while nvidia-smi samples the SM clock every
# 50 ms, and write profiles/<out>.json = per-mode rates at the median clock under load.
set -e
cd "$(dirname "$0")"
OUT=${1:-../../profiles/r02_intpeak.json}
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o intpeak intpeak.cu
cuobjdump -sass intpeak > /tmp/intpeak.sass
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv,noheader,nounits -lms 50 > /tmp/intpeak_clk.csv &
SMI=$!
sleep 0.5
./intpeak 1965 > /tmp/intpeak_nominal.jsonl
kill $SMI || true
python3 - "$OUT" <<'PY'
import json, statistics, sys, subprocess
rows = [json.loads(l) for l in open("/tmp/intpeak_nominal.jsonl")]
clk = []
for ln in open("/tmp/intpeak_clk.csv"):
    p = [x.strip() for x in ln.split(",")]
    try:
        clk.append((float(p[0]), float(p[1]), p[2]))
    except Exception:
        pass
load = [c for c in clk if c[0] > 1000] or clk
med = statistics.median(c[0] for c in load)
smax = max(c[1] for c in clk)
out = {"what": "int32 max-plus instruction mixes, 148 SMs x 4 CTAs x 512 threads, 8 independent "
               "chains per thread (tools/microbench/intpeak.cu); rates at the median SM clock "
               "sampled by nvidia-smi during the run",
       "sm_mhz_median": med, "sm_max_mhz": smax, "clock_samples": len(clk),
       "event_reasons": sorted({c[2] for c in clk}),
       "gpu": subprocess.run(["nvidia-smi", "--query-gpu=name", "--format=csv,noheader"],
                             capture_output=True, text=True).stdout.strip(),
       "modes": {}}
for r in rows:
    scale = 1965.0 / med   # intpeak computed clocks at 1965 MHz
    out["modes"][r["mode"]] = {
        "ms": r["ms"],
        "warp_instr_per_clk_per_smsp": r["warp_instr_per_clk_per_smsp"] * scale,
        "int32_ops_per_clk_per_sm": r["int32_ops_per_clk_per_sm"] * scale,
        "int32_ops_per_s": r["int32_ops_per_s"]}
json.dump(out, open(sys.argv[1], "w"), indent=1)
print(json.dumps(out))
PY
