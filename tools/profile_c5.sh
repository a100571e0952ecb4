#!/bin/bash
# ncu of the C5 batch's intersect / decode-once kernels (one batch, 10K queries, top-1000)
cat > /tmp/c5one.py <<'PY'
import sys; sys.path.insert(0, '.')
from tools.bench_configs import dev_batch
import paper_conf_ppopp_0044ws18_b200 as g
from synth import make_workload
import torch
c, ql, cfg = make_workload("c5")
ix = g.GriffinIndex(c, block_size=128)
run = dev_batch(ix, ql, cfg["k"])
run(); torch.cuda.synchronize(); run(); torch.cuda.synchronize()
PY
timeout 1800 ncu --set full --clock-control none --import-source on -k regex:"intersect_kernel|decode_once" -s 3 -c 3 -o gpurun_out/prof_c5 -f python /tmp/c5one.py > gpurun_out/prof_c5.log 2>&1
tail -3 gpurun_out/prof_c5.log
