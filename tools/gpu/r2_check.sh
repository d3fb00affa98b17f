set -x
python -c "import __graft_entry__ as g; g.build()" 
timeout 300 python bench.py --workload C1 --steps 3 --warmup 3 --cpu-seconds 1 > gpurun_out/b_c1.log 2>&1; echo rc=$?
NESTGPU_DIST_BACKEND=gloo timeout 600 python bench.py --gpus 2 --workload C1 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/b_c1_g2.log 2>&1; echo rc=$?
timeout 600 python bench.py --workload C2 --steps 3 --warmup 3 --cpu-seconds 2 > gpurun_out/b_c2.log 2>&1; echo rc=$?
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 1200 python bench.py > gpurun_out/b_c5.log 2>&1; echo rc=$?
tail -c 3000 gpurun_out/b_c5.log
