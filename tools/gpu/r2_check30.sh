set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/pytest30.log 2>&1; echo rc=$?; tail -3 gpurun_out/pytest30.log
python -c "import __graft_entry__ as g; g.smoke()"
timeout 600 python tools/latency_table.py --skip-c5 --reps 10 --out gpurun_out/r02_latency_s30.jsonl > gpurun_out/latency30.log 2>&1; echo rc=$?
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe30.log 2>&1; cat gpurun_out/latency_probe30.log | cut -c1-150
timeout 600 python tools/time_sort.py
