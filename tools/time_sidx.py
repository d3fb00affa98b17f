"""Time the index build of SF10 Q4 (l_orderkey: key-ordered, sort-free,
EXISTS) and SF1 Q2 for the library in $NESTGPU_LIB: wall clock of
build_index (synchronised), best of 7."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import tpch  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402
from tests.gpu_helpers import load  # noqa: E402
import torch  # noqa: E402

eng = Engine(0, arena_bytes=16 << 30)
out = []
for q, sf, seed in (("q4", 10.0, 5), ("q2", 1.0, 3)):
    t, plan = tpch.flattened(q, sf, seed)
    m0 = eng.mark()
    R, S = load(eng, t)
    best = 1e9
    for _ in range(7):
        m = eng.mark()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        eng.index_for_plan(plan, S)
        torch.cuda.synchronize()
        best = min(best, time.perf_counter() - t0)
        eng.release(m)
    out.append("%s SF%g build_index %.4f ms" % (q, sf, best * 1e3))
    eng.release(m0)
print(os.path.basename(os.environ.get("NESTGPU_LIB", "default")), " | ".join(out))
