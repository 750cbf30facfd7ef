#!/bin/bash
# A/B timing of the sweep's work-distribution knobs on C3/C4 (not the bench)
run() { echo "== $*"; env "$@" python tools/quick_time.py 3 4 2>&1 | cut -c1-110; }
for rep in 1 2; do
run AP_SWEEP_SCHED=static
run AP_SWEEP_MINSIMS=1
run AP_SWEEP_MINSIMS=32
run AP_SWEEP_MINSIMS=128
run AP_SWEEP_MINSIMS=32 AP_SWEEP_UPW=64
run AP_SWEEP_MINSIMS=32 AP_SWEEP_UPW=256
done
