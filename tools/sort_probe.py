"""Build one index over 16M (u32 key, u32 payload) rows -- a single-kernel
target for `ncu -k regex:onesweep` captures of the radix pass."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 16_000_000
rng = np.random.default_rng(0)
eng = Engine(0, arena_bytes=4 << 30)
cols = {"k": eng.load_column(rng.integers(0, 2 ** 31 - 1, n).astype(np.int32)),
        "v": eng.load_column(rng.integers(0, 2 ** 20, n).astype(np.int32))}
for _ in range(2):
    m = eng.mark()
    eng.build_index(cols, ["k"], "v")
    eng.release(m)
print("done")
