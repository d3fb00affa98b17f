set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe3.log 2>&1; echo rc=$?
cat gpurun_out/latency_probe3.log | tail -8
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu3.log 2>&1; echo rc=$?
tail -15 gpurun_out/pytest_gpu3.log
timeout 600 python bench.py --workload C2 --steps 5 --warmup 3 --cpu-seconds 2 --no-side > gpurun_out/b_c2_3.log 2>&1; echo rc=$?
tail -c 600 gpurun_out/b_c2_3.log
