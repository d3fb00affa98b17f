set -x
python -c "import __graft_entry__ as g; g.build()"
python tools/time_filter.py
NESTGPU_FILTER_TWO_PASS=1 python tools/time_filter.py
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tpch.py tests/test_gpu_typej.py tests/test_gpu_multirank.py -x -q > gpurun_out/pytest24.log 2>&1; echo rc=$?; tail -3 gpurun_out/pytest24.log
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe24.log 2>&1; cat gpurun_out/latency_probe24.log
timeout 1500 python tools/cost_model.py --out gpurun_out/r02_cost_model_s24.jsonl > gpurun_out/cost24.log 2>&1; echo rc=$?
