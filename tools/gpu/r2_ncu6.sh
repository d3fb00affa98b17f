set -x
python -c "import __graft_entry__ as g; g.build()"
# launch list of the C5 bench command (1 warm-up, 1 timed step; no side keys): per-launch time + DRAM bytes
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 100 --csv --log-file gpurun_out/r02_launches_C5.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-side --no-cpu-baseline --no-check > gpurun_out/ncu_c5_bench.log 2>&1; echo rc=$?
tail -3 gpurun_out/r02_launches_C5.csv
# per-kernel durations of the SF1 Q2 / C1 index queries (latency diagnosis)
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches_q2.csv python tools/profile_one.py tpch q2 index 1 > gpurun_out/ncu_q2.log 2>&1; echo rc=$?
# one full capture of the '>' MIN nested loop on C5's distributions at |R| = 524288 (x 16M S')
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bnl_kernel -c 1 -o gpurun_out/r02_bnl_c5_min python tools/profile_c5.py 524288 min > gpurun_out/ncu_bnl.log 2>&1; echo rc=$?
ls -la gpurun_out/
