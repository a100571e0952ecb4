#!/bin/bash
# usage: bash profile_run.sh <tag>   (runs on the GPU box)
TAG=${1:-r01}
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -5
timeout 300 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -c 3000 gpurun_out/bench_$TAG.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --latency-queries 5 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:intersect_kernel -s 4 -c 2 -o gpurun_out/prof_$TAG -f python bench.py --steps 1 --warmup 1 --no-cpu-baseline --latency-queries 5 > gpurun_out/ncu_$TAG.log 2>&1
tail -3 gpurun_out/ncu_$TAG.log
ls -la gpurun_out
