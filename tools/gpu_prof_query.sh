# ncu --set full of one batch's intersect + decode-once kernels: CFG, REUSE, TAG
set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
python tools/one_batch.py ${CFG:-c5} ${REUSE:-2} 1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"intersect_kernel|probe_kernel|decode_once" \
  -s ${SKIP:-3} -c ${COUNT:-3} -o gpurun_out/${TAG} -f python tools/one_batch.py ${CFG:-c5} ${REUSE:-2} 3 \
  > gpurun_out/${TAG}.log 2>&1
tail -3 gpurun_out/${TAG}.log
