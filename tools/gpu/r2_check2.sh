set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "exact_int64 or zipf or error_paths or int64 or degenerate or c2_shaped or c1" > gpurun_out/pytest_sel.log 2>&1; echo rc=$?
tail -5 gpurun_out/pytest_sel.log
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe.log 2>&1; echo rc=$?
cat gpurun_out/latency_probe.log | tail -8
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu2.log 2>&1; echo rc=$?
tail -3 gpurun_out/pytest_gpu2.log
