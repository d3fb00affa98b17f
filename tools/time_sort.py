"""Time the index build (S' filter + digit histogram + radix passes) for the
library in $NESTGPU_LIB: 16M int32 keys + int32 payload (C5 S), 38M int64
keys (Q4-like), 60M int32 keys + payload."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402

from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_SORT  # noqa: E402

eng = Engine(0, arena_bytes=8 << 30)
eng.set_profiling(True)
MODES = {"auto": 0}
rng = np.random.default_rng(0)
out = []
for name, k, v in (("1M u32 (18 bits, C2-like)+v32", rng.integers(0, 1 << 18, 1_000_000).astype(np.int32),
                    rng.integers(0, 1 << 20, 1_000_000).astype(np.int32)),
                   ("16M u32+v32", rng.integers(0, 2 ** 31 - 1, 16_000_000).astype(np.int32),
                    rng.integers(0, 2 ** 20, 16_000_000).astype(np.int32)),
                   ("38M u64", (rng.integers(0, 15_000_000, 38_000_000) // 8 * 32).astype(np.int64), None),
                   ("60M u32+v32", rng.integers(0, 2 ** 26, 60_000_000).astype(np.int32),
                    rng.integers(0, 5000, 60_000_000).astype(np.int32)),
                   ("9.1M u64 (38 bits, Q20-like)+v64", (rng.integers(1, 2_000_001, 9_100_000) << 32)
                    + rng.integers(1, 100_001, 9_100_000), rng.integers(1, 50, 9_100_000).astype(np.int64)),
                   ("16M u64 (64 bits)", rng.integers(-2 ** 63, 2 ** 63 - 1, 16_000_000, dtype=np.int64), None),
                   ("6M u32 (18 bits, Q17-like)+v32", rng.integers(0, 200_000, 6_000_000).astype(np.int32),
                    rng.integers(1, 51, 6_000_000).astype(np.int32))):
    m = eng.mark()
    cols = {"k": eng.load_column(k)}
    if v is not None:
        cols["v"] = eng.load_column(v)
    for mname, mode in MODES.items():
        eng.set_option(OPT_SORT, mode)
        best = None
        for _ in range(3):
            m2 = eng.mark()
            eng.build_index(cols, ["k"], "v" if v is not None else None)
            p = eng.last_profile()
            eng.release(m2)
            t = (p["inner_filter"], p["sort"])
            best = t if best is None or sum(t) < sum(best) else best
        out.append("%s [%s] filter %.3f ms sort %.3f ms" % (name, mname, best[0], best[1]))
    eng.set_option(OPT_SORT, 0)
    eng.release(m)
print(os.path.basename(os.environ.get("NESTGPU_LIB", "default")))
print("\n".join(out))

# library baseline on the same inputs: torch.sort (CUB radix sort pairs: key +
# int64 index), CUDA events, best of 5
import torch  # noqa: E402
lib = []
for name, k in (("16M u32 keys (+ int64 idx)", rng.integers(0, 2 ** 31 - 1, 16_000_000).astype(np.int32)),
                ("38M u64-range keys (+ int64 idx)", (rng.integers(0, 15_000_000, 38_000_000) // 8 * 32).astype(np.int64))):
    t = torch.from_numpy(k).cuda()
    best = 1e9
    for _ in range(6):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        torch.sort(t, stable=True)
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    lib.append("%s %.3f ms" % (name, best))
print("torch.sort (CUB):", " | ".join(lib))
