set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
for w in ${WHICH:-c1 c3 c5 codecs}; do
  timeout 1200 python tools/bench_configs.py $w > gpurun_out/${TAG}_$w.jsonl 2> gpurun_out/${TAG}_$w.err
  echo "$w rc=$?"; tail -1 gpurun_out/${TAG}_$w.err
done
