set -x
python -c "import __graft_entry__ as g; g.build()"
python tools/trace_probe.py > gpurun_out/trace20.log 2>&1; grep -A2 -- "---" gpurun_out/trace20.log | tail -9
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe20.log 2>&1; cat gpurun_out/latency_probe20.log
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/pytest20.log 2>&1; echo rc=$?; tail -5 gpurun_out/pytest20.log
