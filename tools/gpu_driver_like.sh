# what the driver runs at round end: reference arm then ours (N=1), timed
set -x
python -c "import __graft_entry__ as e; e.build()"
rm -rf /tmp/griffin_synth
t0=$(date +%s)
python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/${TAG}_ref.json 2> gpurun_out/${TAG}_ref.err
t1=$(date +%s); echo "ref rc=$? wall $((t1-t0)) s"
python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/${TAG}_ours.json 2> gpurun_out/${TAG}_ours.err
t2=$(date +%s); echo "ours rc=$? wall $((t2-t1)) s"
python -c "import __graft_entry__ as e; e.smoke()"
