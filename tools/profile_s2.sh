#!/bin/bash
# usage: bash tools/profile_s2.sh <tag>  (GPU box) — ncu full captures of the
# decode sweep kernel and the two intersect launches of one C2 step.
TAG=${1:-s2}
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:decode_all_kernel -c 1 -o gpurun_out/dec_$TAG -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline --latency-queries 5 --streams 1 > gpurun_out/ncudec_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"intersect_kernel|decode_once" -s 6 -c 3 -o gpurun_out/prof_$TAG -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --latency-queries 5 --streams 1 > gpurun_out/ncu_$TAG.log 2>&1
tail -3 gpurun_out/ncu_$TAG.log gpurun_out/ncudec_$TAG.log
ls -la gpurun_out
