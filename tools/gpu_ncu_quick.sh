# per-kernel metrics of C5 batch 0 (second run) + --set full of the round-1 intersect kernels
# usage (under gpurun): bash tools/gpu_ncu_quick.sh <tag> [full: 0/1]
TAG=$1; FULL=${2:-1}
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/${TAG}_kern.csv \
  -k regex:"intersect_kernel|probe_kernel|decode_once|compact_copy|bm_zero|topk|unit_scan" -s 40 -c 40 \
  python tools/one_batch.py c5 2 3 > gpurun_out/${TAG}_kern.log 2>&1
echo kern_rc=$?
if [ "$FULL" = 1 ]; then
  timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"intersect_kernel" -s 2 -c 2 \
    -o gpurun_out/${TAG}_full -f python tools/one_batch.py c5 2 2 > gpurun_out/${TAG}_full.log 2>&1
  echo full_rc=$?
fi
