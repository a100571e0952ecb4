#!/bin/bash
# usage: bash tools/ab_run.sh <config> <lib1> <lib2> ...   (GPU box) — stage_probe per library
CFG=$1; shift
for L in "$@"; do
  echo "== $L"
  GRIFFIN_LIBRARY=$L timeout 300 python tools/stage_probe.py $CFG 2>&1 | tail -3
done
