set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
python tools/decode_check.py c2 64,128,256,512 2>&1 | tee gpurun_out/r2_dec1.txt
timeout 900 python -m pytest tests -m gpu -x -q -k "decode or encoder or bit_exact or intersect" 2>&1 | tail -15
