# ncu evidence for the current build: launch list of the bench command + --set full of the
# dominant kernels (one C5/C2 batch: decode_once, intersect<1,1>, intersect<1,2>, probe_kernel),
# one GPU; never a multi-rank command.  usage (under gpurun): TAG=x CFGS="c5 c2" bash tools/gpu_evidence.sh
set -x
python -c "import __graft_entry__ as e; e.build()"
for cfg in ${CFGS:-c5 c2}; do
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_$cfg.csv \
     python bench.py --config $cfg --steps 2 --warmup 3 --no-cpu-baseline --latency-queries 5 > /dev/null 2>&1
  echo "launches $cfg rc=$?"
  timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"intersect_kernel|probe_kernel|decode_once" -s 8 -c 4 \
     -o gpurun_out/${TAG}_full_$cfg -f python tools/one_batch.py $cfg 2 4 > gpurun_out/${TAG}_full_$cfg.log 2>&1
  echo "full $cfg rc=$?"; tail -2 gpurun_out/${TAG}_full_$cfg.log
done
