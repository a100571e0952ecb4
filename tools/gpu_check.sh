#!/bin/bash
# GPU-box check: parity tests + bench; summaries printed at the end.
TAG=${1:-x}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider --timeout 240 --timeout-method thread > gpurun_out/tests_$TAG.log 2>&1
timeout 400 python bench.py --no-cpu-baseline > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
echo "== tests: $(tail -1 gpurun_out/tests_$TAG.log)"
grep -E "^(FAILED|E  )" gpurun_out/tests_$TAG.log | head -10
python - <<PY
import json
d=json.load(open("gpurun_out/bench_$TAG.json"))
print("== qps", round(d["value"]), "ms/step", round(d["ms_per_step"],4), "e2e", round(d["e2e"]["value"]))
print("== stages", {k: round(v,4) for k,v in d["stage_ms_per_step"].items()})
print("== roofline", {k: d["roofline"][k] for k in ("kernel","achieved","frac")})
PY
