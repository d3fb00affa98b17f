set -x
python -c "import __graft_entry__ as g; g.build()"
python tools/time_filter.py
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tpch.py tests/test_gpu_typej.py -x -q > gpurun_out/pytest26.log 2>&1; echo rc=$?; tail -3 gpurun_out/pytest26.log
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe26.log 2>&1; cat gpurun_out/latency_probe26.log | cut -c1-200
