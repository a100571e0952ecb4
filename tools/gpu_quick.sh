# quick GPU check: targeted parity tests + default C5 bench (no CPU baseline)
# usage (under gpurun): bash tools/gpu_quick.sh <tag> [pytest -k expr|-] [extra bench args]
TAG=$1; shift
K=${1:-"bitmap or reuse or random or locality"}; [ $# -gt 0 ] && shift
if [ "$K" != "-" ]; then
  timeout 400 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/${TAG}_pytest.log 2>&1
  echo pytest_rc=$? >> gpurun_out/${TAG}_pytest.log
fi
timeout 700 python bench.py --no-cpu-baseline "$@" > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
echo bench_rc=$?
