# A/B of alternate library builds (ab/libgriffin_<tag>.so) vs the current one with stage_probe
set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
for cfg in ${CFGS:-c2 c5}; do
  for lib in current ${LIBS}; do
    if [ "$lib" = current ]; then python tools/stage_probe.py $cfg 2>&1 | sed "s/^/current /" | tee -a gpurun_out/${TAG}_ab.txt;
    else GRIFFIN_LIBRARY=ab/libgriffin_$lib.so python tools/stage_probe.py $cfg 2>&1 | sed "s/^/$lib /" | tee -a gpurun_out/${TAG}_ab.txt; fi
  done
done
