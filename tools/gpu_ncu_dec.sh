# ncu --set full of the decode-only sweep kernel (one launch, after warm-up)
set -x
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
python tools/decode_check.py c2 128 > /dev/null   # warm the synth cache
ncu --set full --clock-control none --import-source on -k regex:decode_all -s 2 -c 1 \
    -o gpurun_out/${TAG:-dec} python tools/decode_check.py c2 128 > gpurun_out/${TAG:-dec}.log 2>&1
tail -3 gpurun_out/${TAG:-dec}.log
