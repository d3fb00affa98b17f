"""Small workload touching every kernel, for compute-sanitizer runs:
filter (ordered / unordered), sort + histogram, range (short, long, prefix
aggregates), nested loop (all agg kinds, both R-block shapes), dedup (iota /
group), finalize, gather, minmax, type-J collections + IN + materialise,
cost-model calibration (fills), and the radix-sort variants (pre-narrowed
64-bit keys, 9-bit digit passes, keys without payload)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from datagen import make_plan, query1  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200 import Engine  # noqa: E402
from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_BNL_SHAPE  # noqa: E402

eng = Engine(0, arena_bytes=512 << 20)
t = query1.random_small(1, n_r=20011, n_s=30011, key_hi=600, val_lo=-50, val_hi=50, null_frac=0.1)
R, S = eng.load_table(t["R"], t.get("R_valid")), eng.load_table(t["S"], t.get("S_valid"))
bad = 0
for mode in ("bnl", "bnl_full", "index"):
    for op in ("=", "!=", "<", ">="):
        for agg in ("min", "max", "sum", "count", "avg", "exists"):
            for dedup in (False, True):
                plan = make_plan(op, agg, "<=", outer_preds=[{"col": "col3", "op": "<=", "lit": 1}],
                                 inner_preds=[{"col": "col3", "op": "!=", "rhs": "col2"}])
                idx = eng.index_for_plan(plan, S) if mode == "index" else -1
                eng.set_option(OPT_BNL_SHAPE, 1 if mode == "bnl_full" else 0)
                g = eng.result_to_numpy(eng.exec(plan, R, S, index=idx, emit_all=True, dedup=dedup))
                ref = oracle.evaluate(t, plan)
                m = ref["in_rp"].astype(bool)
                ok = np.array_equal(g["row"], ref["row"][m]) and np.array_equal(g["value"], ref["value"][m])
                bad += not ok
big = {"k": np.zeros(8, np.int64), "v": np.arange(8, dtype=np.int64)}
S2 = eng.load_table(big, dtypes={"v": "decimal"})
R2 = eng.load_table({"k": np.zeros(3, np.int64), "x": np.zeros(3, np.int64)})
res = eng.exec(make_plan("=", "sum", "<", outer_key=["k"], inner_key=["k"], agg_col="v", outer_cmp_col="x"), R2, S2)
eng.gather_column(R2["x"], res)
eng.set_option(OPT_BNL_SHAPE, 0)
# type-J collections, IN over them, materialisation
plan = make_plan("=", "min", "=", inner_preds=[{"col": "col3", "op": ">=", "lit": 1}])
idx = eng.build_index(S, ["col1"], payload="col2", inner_preds=plan["inner_preds"])
coll = eng.exec_collect(plan, R, S, idx)
c = eng.collection_to_numpy(coll)
ref = oracle.collect(t, plan)
bad += not np.array_equal(np.diff(c["offsets"]), ref["lens"][ref["in_rp"].astype(bool)])
eng.result_to_numpy(eng.collection_in(coll, R["col2"], emit_all=True))
col = eng.column_from_device(coll.d_values, coll.n_values, "int32")
# sort variants: 64-bit keys pre-narrowed to 32 bits by the filter, 18-bit
# keys (9-bit digit passes), keys without payload (4-byte items), all vs numpy
rng = np.random.default_rng(5)
for keys, dt, pay in ((rng.integers(0, 1 << 29, 70001) + (7 << 40), "int64", True),
                      (rng.integers(0, 1 << 18, 70001), "int32", True),
                      (rng.integers(0, 1 << 26, 90001), "int32", False)):
    cols = {"k": keys, "v": np.arange(len(keys))} if pay else {"k": keys}
    T = eng.load_table(cols, dtypes={"k": dt, "v": "int32"} if pay else {"k": dt})
    ix = eng.build_index(T, ["k"], "v" if pay else None)
    info = eng.index_info(ix)
    kb = info["key_bytes"]
    import torch
    got = eng.arena_view(info["d_keys"], len(keys) * kb).view(torch.int64 if kb == 8 else torch.int32).cpu().numpy()
    enc = (keys.astype(np.int64).view(np.uint64) ^ np.uint64(1 << 63)) if kb == 8 else \
        (keys.astype(np.int32).view(np.uint32) ^ np.uint32(1 << 31))
    bad += not np.array_equal(got.view(enc.dtype), np.sort(enc))
eng.cost_calibrate(1 << 16)
print("sanitize workload done, mismatches:", bad)
sys.exit(1 if bad else 0)
