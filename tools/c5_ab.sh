#!/bin/bash
# C5 heuristic kernel A/B over library variants, interleaved.  usage: c5_ab.sh LIB...
for round in 1 2; do
  for lib in "$@"; do
    printf "%s " "$(basename $lib)"
    AP_LIB_PATH=$lib python tools/c5_once.py 3 2>&1 | grep -o "kernel [0-9.]* ms" | tr '\n' ' '
    echo
  done
done
