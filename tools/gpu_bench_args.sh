# A/B of bench.py arguments on one box: each "name=args" pair -> gpurun_out/<tag>_<name>.json
# usage (under gpurun): bash tools/gpu_bench_args.sh <tag> "name1=--x 1" "name2=--y 2" ...
TAG=$1; shift
for pair in "$@"; do
  name=${pair%%=*}; args=${pair#*=}
  timeout 700 python bench.py --no-cpu-baseline --latency-queries 100 $args \
    > gpurun_out/${TAG}_$name.json 2> gpurun_out/${TAG}_$name.err
  echo "$name rc=$?"
done
