# A/B of library builds on one box: the in-tree build, then each ab/libgriffin_<v>.so
# usage (under gpurun): bash tools/gpu_ab_libs.sh <tag> "<v1> <v2> ..." [extra bench args]
TAG=$1; VS=$2; shift 2
for v in main $VS; do
  if [ "$v" = main ]; then LIBENV=""; else LIBENV="GRIFFIN_LIBRARY=$PWD/ab/libgriffin_$v.so"; fi
  env $LIBENV timeout 700 python bench.py --no-cpu-baseline --latency-queries 100 "$@" \
    > gpurun_out/${TAG}_$v.json 2> gpurun_out/${TAG}_$v.err
  echo "$v rc=$?"
done
