#!/bin/bash
# usage: bash tools/prof_ik.sh <tag>  (GPU box) — ncu full capture of one C2 step's
# decode_once + intersect launches (1 stream).
TAG=${1:-x}
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"intersect_kernel|decode_once" -s 6 -c 3 -o gpurun_out/prof_$TAG -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --latency-queries 5 --streams 1 > gpurun_out/ncu_$TAG.log 2>&1
tail -2 gpurun_out/ncu_$TAG.log
