"""Build SF10 Q20's index once (S' filter + sort) -- a target for an ncu
capture of the S' filter (filter_tma_kernel)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import tpch  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402
from tests.gpu_helpers import load  # noqa: E402

q = sys.argv[1] if len(sys.argv) > 1 else "q20"
t, plan = tpch.flattened(q, 10.0, 5)
eng = Engine(0, arena_bytes=16 << 30)
R, S = load(eng, t)
for _ in range(2):
    m = eng.mark()
    eng.index_for_plan(plan, S)
    eng.release(m)
print("done")
