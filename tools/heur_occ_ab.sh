#!/bin/bash
# C5 heuristic pool: CTAs/SM A/B (AP_HEUR_OCC), interleaved on one box.
for round in 1 2; do
  for occ in 4 3 2 1; do
    echo "occ=$occ round=$round"
    AP_HEUR_OCC=$occ python tools/c5_once.py 4 2>&1 | grep search | tail -3
  done
done
