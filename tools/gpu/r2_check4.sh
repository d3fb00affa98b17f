set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_multirank.py tests/test_bench_cpu.py -x -q -m gpu > gpurun_out/pytest_mr4.log 2>&1; echo rc=$?
tail -15 gpurun_out/pytest_mr4.log
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe4.log 2>&1; echo rc=$?
cat gpurun_out/latency_probe4.log | tail -8
NESTGPU_DIST_BACKEND=gloo timeout 600 python bench.py --gpus 2 --workload C2 --steps 3 --warmup 3 --no-cpu-baseline --no-side > gpurun_out/b_c2_g2.log 2>&1; echo rc=$?
tail -c 1500 gpurun_out/b_c2_g2.log
