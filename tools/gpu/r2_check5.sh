set -x
python -c "import __graft_entry__ as g; g.build()"
python tools/trace_probe.py > gpurun_out/trace5.log 2>&1; grep -A2 -- "---" gpurun_out/trace5.log | tail -12
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe5.log 2>&1; echo rc=$?
cat gpurun_out/latency_probe5.log | tail -8
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu5.log 2>&1; echo rc=$?
tail -15 gpurun_out/pytest_gpu5.log
timeout 300 python tools/time_sort.py > gpurun_out/time_sort5.log 2>&1; cat gpurun_out/time_sort5.log
