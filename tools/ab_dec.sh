#!/bin/bash
# usage: bash tools/ab_dec.sh lib1 lib2 ...  (GPU box) — C2 stage probe + decode sweeps at B = 64..512
for L in "$@"; do
  echo "== $L"
  GRIFFIN_LIBRARY=$L timeout 300 python tools/stage_probe.py c2 2>&1 | tail -2
  for B in 64 256 512; do
    PROBE_B=$B GRIFFIN_LIBRARY=$L timeout 300 python tools/stage_probe.py c2 2>&1 | tail -1 | sed "s/^/B=$B /"
  done
done
