"""One index-path query (build_index + exec + result_to_host), repeated, for
an ncu launch list of its kernels: python tools/query_launches.py C2 = min
| q2 [sf].  Prints nothing useful itself; run it under
`ncu --metrics gpu__time_duration.sum`."""
import os
import sys

import numpy as np  # noqa: F401

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
eng = Engine(0, arena_bytes=4 << 30)
R, S = load(eng, tabs)
for rep in range(int(os.environ.get("REPS", "3"))):
    m = eng.mark()
    idx = eng.index_for_plan(plan, S)
    res = eng.exec(plan, R, S, index=idx)
    eng.result_to_numpy(res)
    eng.release(m)
print("done")
