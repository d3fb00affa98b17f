set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python tools/cost_model.py --out gpurun_out/r02_cost_model.jsonl > gpurun_out/cost23.log 2>&1; echo rc=$?; tail -c 2000 gpurun_out/cost23.log
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/pytest23.log 2>&1; echo rc=$?; tail -5 gpurun_out/pytest23.log
python -c "import __graft_entry__ as g; g.smoke()"
