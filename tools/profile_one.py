"""Run one plan twice (for `ncu --set full` captures of single kernels).

  python tools/profile_one.py <op> <agg> <mode> [C1|C2|C5]     Query-1 family
  python tools/profile_one.py tpch <q2|q17|q4|q20> <mode> [SF]   TPC-H-shaped
  NESTGPU_DEDUP=1 runs the plan with caching.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from datagen import make_plan, query1, tpch  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402

if sys.argv[1] == "tpch":
    q, mode = sys.argv[2], sys.argv[3]
    sf = float(sys.argv[4]) if len(sys.argv) > 4 else 10.0
    t, plan = tpch.QUERIES[q](tpch.base_tables(sf, 5))
else:
    op, agg, mode = sys.argv[1], sys.argv[2], sys.argv[3]
    wl = sys.argv[4] if len(sys.argv) > 4 else "C2"
    t = query1.config(wl)
    plan = make_plan(op, agg, "=")
eng = Engine(0, arena_bytes=24 << 30)
R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
eng.set_profiling(True)
for _ in range(2):
    idx = eng.index_for_plan(plan, S) if mode == "index" else -1
    res = eng.exec(plan, R, S, index=idx, dedup=os.environ.get("NESTGPU_DEDUP") == "1")
print("survivors", res.n_rows, "launches", eng.launch_count(), eng.last_profile())
