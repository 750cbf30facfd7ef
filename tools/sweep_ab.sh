#!/bin/bash
# C4 FULL sweep kernel A/B over library variants (tools/quick_time.py 4), interleaved.
for round in 1 2; do
  for lib in "$@"; do
    printf "%s " "$(basename $lib)"
    AP_LIB_PATH=$lib python tools/quick_time.py 4 2>&1 | tail -1
  done
done
