"""Time the nested-loop kernel on C2 plans for the library in $NESTGPU_LIB."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import make_plan, query1  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "C2"
t = query1.config(wl)
eng = Engine(0, arena_bytes=2 << 30)
R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
eng.set_profiling(True)
out = []
for op, agg in ((">", "min"), (">", "count"), ("!=", "count"), ("<", "sum"), (">", "exists")):
    plan = make_plan(op, agg, "=")
    ms = []
    for _ in range(3):
        eng.exec(plan, R, S)
        ms.append(eng.last_profile()["subquery"])
    out.append("%s %s %.2f" % (op, agg, min(ms)))
print(os.path.basename(os.environ.get("NESTGPU_LIB", "default")), " | ".join(out))
