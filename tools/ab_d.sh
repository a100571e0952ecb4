bash tools/ab_run.sh c2 abx/libgriffin_d8.so
echo "== D=4 minb4"; GRIFFIN_TUNE_D=4 GRIFFIN_LIBRARY=abx/libgriffin_mb4.so timeout 300 python tools/stage_probe.py c2 2>&1 | tail -2
echo "== D=5 minb4"; GRIFFIN_TUNE_D=5 GRIFFIN_LIBRARY=abx/libgriffin_mb4.so timeout 300 python tools/stage_probe.py c2 2>&1 | tail -2
echo "== D=8 minb4"; GRIFFIN_LIBRARY=abx/libgriffin_mb4.so timeout 300 python tools/stage_probe.py c2 2>&1 | tail -2
echo "== D=6 minb3"; GRIFFIN_TUNE_D=6 GRIFFIN_LIBRARY=abx/libgriffin_d8.so timeout 300 python tools/stage_probe.py c2 2>&1 | tail -2
echo "== D=12 minb3"; GRIFFIN_TUNE_D=12 GRIFFIN_LIBRARY=abx/libgriffin_d8.so timeout 300 python tools/stage_probe.py c2 2>&1 | tail -2
