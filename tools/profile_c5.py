"""One nested-loop launch on C5's distributions (keys U[0,2^31-1), values
U[0,2^20), |S| = 16M) with a reduced |R| -- a target for `ncu --set full`
captures of bnl_kernel (a full C5 launch is 28 s, x ~40 replays).
usage: python tools/profile_c5.py [n_r] [min|count]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import make_plan, query1  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402

n_r = int(sys.argv[1]) if len(sys.argv) > 1 else 524288
agg = sys.argv[2] if len(sys.argv) > 2 else "min"
t = query1.config("C5", n_r=n_r)
eng = Engine(0, arena_bytes=4 << 30)
R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
res = eng.exec(make_plan(">", agg, "="), R, S)
print("survivors", res.n_rows)
