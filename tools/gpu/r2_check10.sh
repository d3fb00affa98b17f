set -x
python -c "import __graft_entry__ as g; g.build()"
python tools/time_filter.py
NESTGPU_LIB=vlib/b16.so python tools/time_filter.py
NESTGPU_LIB=vlib/b4.so python tools/time_filter.py
NESTGPU_FILTER_TWO_PASS=1 python tools/time_filter.py
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c1 or null or degenerate or random or predicates or c2_shaped or composite" > gpurun_out/pytest10.log 2>&1; echo rc=$?; tail -3 gpurun_out/pytest10.log
