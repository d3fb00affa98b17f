"""Diagnose: exact int64 sums on the index path with exec graphs on / off."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from datagen import make_plan, PLAN_OPS  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine, NestGPUError  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_GRAPHS  # noqa: E402
from tests.gpu_helpers import run  # noqa: E402

eng = Engine(0, arena_bytes=1 << 30)
rng = np.random.default_rng(77)
pairs = 6007
A = (1 << 62) + (1 << 61)
keys = np.repeat(np.arange(pairs, dtype=np.int64) * 3, 2)
vals = np.empty(2 * pairs, np.int64)
vals[0::2] = A + rng.integers(-1000, 1000, pairs)
vals[1::2] = -A + rng.integers(-1000, 1000, pairs)
perm = rng.permutation(2 * pairs)
n_r = 4001
t = {"R": {"col1": rng.integers(-5, 3 * pairs + 5, n_r).astype(np.int64),
           "col2": rng.integers(-3000, 3000, n_r).astype(np.int64)},
     "S": {"col1": keys[perm], "col2": vals[perm]}}
dt = {"R": {"col1": "int64", "col2": "int64"}, "S": {"col1": "int64", "col2": "decimal"}}
for graphs in (0, 1):
    eng.set_option(OPT_GRAPHS, graphs)
    for mode in ("bnl", "index"):
        for corr_op in PLAN_OPS:
            for agg, outer in (("sum", "<"), ("avg", ">=")):
                plan = make_plan(corr_op, agg, outer)
                ref = oracle.evaluate(t, plan)
                try:
                    g = run(eng, t, plan, mode, emit_all=True, dtypes=dt)
                    m = ref["in_rp"].astype(bool)
                    ok = np.array_equal(g["value"], ref["value"][m]) and np.array_equal(g["valid"].astype(np.int64), ref["valid"][m].astype(np.int64))
                    print(graphs, mode, corr_op, agg, "ok" if ok else "MISMATCH")
                except NestGPUError as e:
                    print(graphs, mode, corr_op, agg, "ERROR", e)
