"""Run one plan of the C2 workload once (for `ncu --set full` captures of a
single kernel).  Usage: python tools/profile_one.py [op] [agg] [mode] [workload]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from datagen import make_plan, query1  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402

op = sys.argv[1] if len(sys.argv) > 1 else ">"
agg = sys.argv[2] if len(sys.argv) > 2 else "min"
mode = sys.argv[3] if len(sys.argv) > 3 else "bnl"
wl = sys.argv[4] if len(sys.argv) > 4 else "C2"
t = query1.config(wl)
eng = Engine(0, arena_bytes=2 << 30)
R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
plan = make_plan(op, agg, "=")
for _ in range(2):
    idx = eng.index_for_plan(plan, S) if mode == "index" else -1
    res = eng.exec(plan, R, S, index=idx)
print("survivors", res.n_rows, "launches", eng.launch_count())
