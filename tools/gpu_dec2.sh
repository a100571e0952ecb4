set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
python tools/decode_check.py c2 64,128,256,512 2>&1 | tee gpurun_out/${TAG}_dec.txt
ncu --set full --clock-control none --import-source on -k regex:decode_all -s 2 -c 1 \
    -o gpurun_out/${TAG} python tools/decode_check.py c2 128 > gpurun_out/${TAG}.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "decode or encoder or bit_exact or intersect" 2>&1 | tail -5
