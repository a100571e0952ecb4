# A/B of env-var variants with stage_probe: VARS="NAME=a NAME=b" CFGS="c2 c5"
set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
for cfg in ${CFGS:-c2 c5}; do
  for v in ${VARS}; do
    env $v python tools/stage_probe.py $cfg 2>&1 | sed "s/^/$v /" | tee -a gpurun_out/${TAG}_ab.txt
  done
done
if [ -n "$TESTS" ]; then timeout 900 python -m pytest tests -m gpu -q -x -k "$TESTS" 2>&1 | tail -3; fi
