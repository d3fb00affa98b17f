"""Time the R' (ordered, one pass) filter for the library in $NESTGPU_LIB:
SF10 Q4's outer filter (15M orders, date window 3.8 %, int64 keys) and
C5's R' (16M rows, no predicate); device time of the exec stages from
nestgpu_last_profile, best of 5."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import make_plan, query1, tpch  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402
from tests.gpu_helpers import load  # noqa: E402

eng = Engine(0, arena_bytes=16 << 30)
eng.set_profiling(True)
out = []
t4, p4 = tpch.flattened("q4", 10.0, 5)
t2, p2 = tpch.flattened("q2", 1.0, 3)
for name, t, plan in (("Q4 SF10", t4, p4), ("C5", query1.config("C5"), make_plan("=", "count", "=")),
                      ("Q2 SF1", t2, p2)):
    m0 = eng.mark()
    R, S = load(eng, t)
    idx = eng.index_for_plan(plan, S)
    best = {}
    for _ in range(5):
        m = eng.mark()
        eng.exec(plan, R, S, index=idx)
        p = eng.last_profile()
        for k in ("outer_filter", "subquery", "finalize"):
            best[k] = min(best.get(k, 1e9), p[k])
        eng.release(m)
    out.append("%s R' filter %.4f ms probe %.4f finalize %.4f" % (name, best["outer_filter"], best["subquery"],
                                                                   best["finalize"]))
    eng.release(m0)
print(os.path.basename(os.environ.get("NESTGPU_LIB", "default")), " | ".join(out))
