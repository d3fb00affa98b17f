"""Device time of the indexed subquery stage (a5 + a6: binary search + range
aggregate) for the library in $NESTGPU_LIB: C2 '=' MIN / COUNT / '<' MIN
(index path), SF1 Q2, SF1 Q17; best of 7 execs over one prebuilt index."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import make_plan, query1, tpch  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402
from tests.gpu_helpers import load  # noqa: E402

eng = Engine(0, arena_bytes=8 << 30)
eng.set_profiling(True)
c2 = query1.config("C2")
cases = [("C2 = min", c2, make_plan("=", "min", "=")), ("C2 = count", c2, make_plan("=", "count", "=")),
         ("C2 < min", c2, make_plan("<", "min", "="))]
for q in ("q2", "q17"):
    t, p = tpch.flattened(q, 1.0, 3)
    cases.append(("SF1 " + q, t, p))
out = []
for name, t, plan in cases:
    m0 = eng.mark()
    R, S = load(eng, t)
    idx = eng.index_for_plan(plan, S)
    best = 1e9
    for _ in range(7):
        m = eng.mark()
        eng.exec(plan, R, S, index=idx)
        best = min(best, eng.last_profile()["subquery"])
        eng.release(m)
    out.append("%s %.4f" % (name, best))
    eng.release(m0)
print(os.path.basename(os.environ.get("NESTGPU_LIB", "default")), " | ".join(out))
