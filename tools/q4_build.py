"""Build SF10 Q4's index twice (key-ordered: ordered count pass + ballot-fed
write pass, no sort) -- a target for ncu captures of those launches."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import tpch  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402
from tests.gpu_helpers import load  # noqa: E402

t, plan = tpch.flattened("q4", 10.0, 5)
eng = Engine(0, arena_bytes=16 << 30)
R, S = load(eng, t)
for _ in range(2):
    m = eng.mark()
    eng.index_for_plan(plan, S)
    eng.release(m)
print("done")
