#!/bin/bash
# usage: bash tools/round_evidence.sh <tag>  (GPU box) — the round's evidence set:
# GPU tests, the bench line, the ncu launch list of the bench command, ncu --set
# full captures of the C2 step's decode_once/intersect launches and of the
# decode sweep.  Summarise here with tools/ncu_summary.py / tools/launch_table.py.
TAG=${1:-x}
mkdir -p gpurun_out
timeout 1300 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=5 > gpurun_out/tests_$TAG.log 2>&1
echo "== tests: $(tail -1 gpurun_out/tests_$TAG.log)"
grep -E "^(FAILED|E  )" gpurun_out/tests_$TAG.log | head -10
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -c 400 gpurun_out/bench_$TAG.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --latency-queries 5 --streams 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"intersect_kernel|decode_once" -s 6 -c 3 -o gpurun_out/prof_$TAG -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --latency-queries 5 --streams 1 > gpurun_out/ncu_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:decode_all_kernel -c 1 -o gpurun_out/dec_$TAG -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline --latency-queries 5 --streams 1 > gpurun_out/ncudec_$TAG.log 2>&1
ls -la gpurun_out | tail -8
