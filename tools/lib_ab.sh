#!/bin/bash
# A/B of library variants on one box, interleaved: C5 heuristic kernel (tools/c5_once.py)
# and ap_eval_batch T + master on C4 and C5 (tools/eval_time.py).  usage: lib_ab.sh LIB...
for round in 1 2; do
  for lib in "$@"; do
    echo "== $lib round $round"
    AP_LIB_PATH=$lib python tools/c5_once.py 4 2>&1 | grep search | tail -3
    AP_LIB_PATH=$lib python tools/eval_time.py 4 22 2>&1 | tail -2
    AP_LIB_PATH=$lib python tools/eval_time.py 5 20 2>&1 | tail -1
  done
done
