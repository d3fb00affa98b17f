"""Wall time of the first '=' MIN exec over a fresh index (it builds the
per-key group aggregates, seg_onepass_kernel) for run-length extremes:
16M keys all equal (one run), Zipf-like hot keys, and short runs."""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from datagen import make_plan  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402
import torch  # noqa: E402

eng = Engine(0, arena_bytes=8 << 30)
rng = np.random.default_rng(1)
n = 16_000_000
cases = {"all equal": np.full(n, 7, np.int32),
         "zipf": np.minimum(rng.zipf(1.3, n), 1 << 20).astype(np.int32),
         "short runs": rng.integers(0, 1 << 22, n).astype(np.int32)}
plan = make_plan("=", "min", "=")
out = []
for name, k in cases.items():
    m0 = eng.mark()
    S = eng.load_table({"col1": k, "col2": rng.integers(-1000, 1000, n).astype(np.int32)})
    R = eng.load_table({"col1": k[:1000].copy(), "col2": np.zeros(1000, np.int32)})
    best = [1e9, 1e9]
    for _ in range(3):
        m = eng.mark()
        idx = eng.index_for_plan(plan, S)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        eng.exec(plan, R, S, index=idx)          # builds the group aggregates
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        eng.exec(plan, R, S, index=idx)          # reuses them
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        best = [min(best[0], t1 - t0), min(best[1], t2 - t1)]
        eng.release(m)
    out.append("%s: first exec %.3f ms, second %.3f ms" % (name, best[0] * 1e3, best[1] * 1e3))
    eng.release(m0)
print(" | ".join(out))
