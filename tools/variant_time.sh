#!/bin/bash
# A/B timing of library build variants (build/var/libap_*.so) on C3/C4 (not the bench)
for rep in 1 2; do
for lib in build/var/libap_*.so; do
  echo "== $lib"
  AP_LIB_PATH=$lib python tools/quick_time.py "$@" 2>&1 | cut -c1-120
done
done
