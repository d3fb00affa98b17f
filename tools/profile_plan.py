"""Per-stage device times (nestgpu_last_profile) of one TPC-H-shaped or
Query-1 plan under each strategy -- a diagnosis helper.
usage: python tools/profile_plan.py q17 [sf] | C2 '<' min"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import make_plan, query1, tpch  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402
from tests.gpu_helpers import load  # noqa: E402

name = sys.argv[1]
if name.startswith("C"):
    tabs = query1.config(name)
    plan = make_plan(sys.argv[2], sys.argv[3], "=")
else:
    tabs, plan = tpch.flattened(name, float(sys.argv[2]) if len(sys.argv) > 2 else 1.0, 3)
eng = Engine(0, arena_bytes=16 << 30)
R, S = load(eng, tabs)
eng.set_profiling(True)
for use_index in (False, True):
    for dedup in (False, True):
        for rep in range(3):
            m = eng.mark()
            idx = eng.index_for_plan(plan, S) if use_index else -1
            res = eng.exec(plan, R, S, index=idx, dedup=dedup)
            p = eng.last_profile()
            eng.release(m)
        print("index" if use_index else "loop ", "dedup" if dedup else "     ", "evals", res.n_evaluated,
              " ".join("%s=%.4f" % (k, v) for k, v in p.items()))
