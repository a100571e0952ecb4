set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
for s in ${STREAMS:-3}; do
  timeout 900 python bench.py --config ${CFG:-c5} --streams $s --steps ${STEPS:-20} --warmup 3 --cpu-budget 6 \
    > gpurun_out/${TAG}_s$s.json 2> gpurun_out/${TAG}_s$s.err
  tail -2 gpurun_out/${TAG}_s$s.err
  nvidia-smi --query-gpu=memory.used,memory.total --format=csv
done
