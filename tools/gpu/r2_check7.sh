set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tpch.py -x -q > gpurun_out/pytest7.log 2>&1; echo rc=$?
tail -5 gpurun_out/pytest7.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches_q2_b.csv python tools/profile_one.py tpch q2 index 1 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:filter_rp --csv --log-file gpurun_out/r02_rp_c5.csv python tools/profile_one.py ">" min bnl C2 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:filter --csv --log-file gpurun_out/r02_filter_q4.csv python tools/profile_one.py tpch q4 index 10 > /dev/null 2>&1
timeout 300 python tools/latency_probe.py --runs 200 > gpurun_out/latency_probe7.log 2>&1; cat gpurun_out/latency_probe7.log
timeout 300 python tools/latency_table.py --skip-c5 --reps 10 --out gpurun_out/r02_latency_s7.jsonl > gpurun_out/latency7.log 2>&1; tail -20 gpurun_out/latency7.log
