# A/B of bench.py variants on one box; each line -> gpurun_out/${TAG}_<cfg>_<variant>.json
set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
for cfg in ${CFGS:-c2 c5}; do
  for v in ${VARIANTS:-auto off}; do
    timeout 900 python bench.py --config $cfg --reuse $v --steps ${STEPS:-10} --warmup 3 --cpu-budget 6 \
      > gpurun_out/${TAG}_${cfg}_${v}.json 2> gpurun_out/${TAG}_${cfg}_${v}.err
    tail -2 gpurun_out/${TAG}_${cfg}_${v}.err
  done
done
