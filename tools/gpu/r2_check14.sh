set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "graph_replay or c1 or degenerate" > gpurun_out/pytest14a.log 2>&1; echo rc=$?; tail -15 gpurun_out/pytest14a.log
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe14.log 2>&1; cat gpurun_out/latency_probe14.log
NESTGPU_GRAPHS=0 timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe14_nog.log 2>&1; cat gpurun_out/latency_probe14_nog.log
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest14.log 2>&1; echo rc=$?; tail -5 gpurun_out/pytest14.log
