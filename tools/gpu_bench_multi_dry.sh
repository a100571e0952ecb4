# The N>1 bench paths on a one-GPU box: 2 ranks share GPU 0 over gloo
set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
for mode in "--exchange allgather" "--exchange sliced" "--shard-mode replicate"; do
  tag=$(echo $mode | tr -d ' -')
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
    bench.py --gpus 2 --config ${CFG:-c2} --steps 6 --warmup 3 --cpu-budget 4 --dist-backend gloo $mode \
    > gpurun_out/${TAG}_$tag.json 2> gpurun_out/${TAG}_$tag.err
  echo "rc=$? $mode"; tail -2 gpurun_out/${TAG}_$tag.err
done
