#!/bin/bash
# A/B of the pruned mode's units-per-warp (lane range length) on C3/C4 (not the bench)
for u in ${UPWS:-1 2 4 8 16 32 64}; do
  echo "== AP_SWEEP_UPW=$u"
  AP_SWEEP_UPW=$u python tools/quick_modes.py 3 4 2>&1 | grep "mode 2"
done
