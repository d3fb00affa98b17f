python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/r02_ref_C5.log 2>&1; echo ref rc=$?
timeout 2400 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r02_bench_C5_full.log 2>&1; echo bench rc=$?
tail -c 600 gpurun_out/r02_ref_C5.log
tail -c 3500 gpurun_out/r02_bench_C5_full.log
