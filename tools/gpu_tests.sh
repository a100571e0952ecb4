# the GPU parity suite (+ smoke); log -> gpurun_out/${TAG}_pytest.log
python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()"
timeout ${LIMIT:-1500} python -m pytest tests -m gpu -q -x ${PYARGS} > gpurun_out/${TAG}_pytest.log 2>&1
echo "pytest rc=$?"
tail -5 gpurun_out/${TAG}_pytest.log
python -c "import __graft_entry__ as e; e.smoke()" 2>&1 | tail -2
