"""Small workload touching every kernel, for compute-sanitizer runs:
filter (ordered / unordered), sort + histogram, range (short, long, prefix
aggregates), nested loop (all agg kinds, both R-block shapes), dedup (iota /
group), finalize, gather, minmax, type-J collections + IN + materialise,
cost-model calibration (fills), the radix-sort variants (pre-narrowed
64-bit keys, 9-bit digit passes, keys without payload), and (round 2) the
exact split SUM/AVG, the one-launch ordered R' filter with and without
predicates, group aggregates, staged small results and a window put; the
key-ordered index build and the MSD bucket sort experiment (session 2)."""
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
# round 2: exact split SUM/AVG of 64-bit payloads (both kernels), the
# ordered R' filter without predicates, '=' MIN over a large index (group
# aggregates), a result stored into a peer-gather window
A = (1 << 62) + (1 << 61)
keys = np.repeat(np.arange(3001, dtype=np.int64) * 3, 2)
vals = np.empty(6002, np.int64)
vals[0::2], vals[1::2] = A + rng.integers(-9, 9, 3001), -A + rng.integers(-9, 9, 3001)
perm = rng.permutation(6002)
tw = {"R": {"col1": rng.integers(-3, 9010, 5003).astype(np.int64), "col2": rng.integers(-99, 99, 5003).astype(np.int64)},
      "S": {"col1": keys[perm], "col2": vals[perm]}}
Rw = eng.load_table(tw["R"], dtypes={"col1": "int64", "col2": "int64"})
Sw = eng.load_table(tw["S"], dtypes={"col1": "int64", "col2": "decimal"})
for op in ("=", ">", "!="):
    for agg in ("sum", "avg"):
        plan = make_plan(op, agg, "<")
        for mode in ("bnl", "index"):
            idx = eng.index_for_plan(plan, Sw) if mode == "index" else -1
            g = eng.result_to_numpy(eng.exec(plan, Rw, Sw, index=idx, emit_all=True))
            ref = oracle.evaluate(tw, plan)
            bad += not np.array_equal(g["value"], ref["value"][ref["in_rp"].astype(bool)])
tn = query1.tables(n_r=70001, n_s=90001, key_hi=5000, val_hi=50, seed=9)
Rn, Sn = eng.load_table(tn["R"]), eng.load_table(tn["S"])
plan = make_plan("=", "min", "=")
res = eng.exec(plan, Rn, Sn, index=eng.index_for_plan(plan, Sn))
win, _ = eng.window_create(res.n_rows + 5)
eng.result_put(res, win, res.n_rows + 5, 0)
er, ev = oracle.survivors(oracle.evaluate(tn, plan))
wi, wv = eng.window_tensors(win, res.n_rows + 5, res.n_rows)
bad += not (np.array_equal(wi.cpu().numpy(), er) and np.array_equal(wv.cpu().numpy(), ev))
eng.window_free(win)
# round 2, session 2: the key-ordered (sort-free) index build with and
# without inner predicates, and the MSD bucket sort experiment
# (NESTGPU_OPT_SORT = 2: group histograms, column scan, partition, finish)
from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_SORT  # noqa: E402
ko = np.sort(rng.integers(-5000, 5000, 50011)).astype(np.int64)
to = {"R": {"col1": rng.integers(-5010, 5010, 7001).astype(np.int64), "col2": rng.integers(-50, 50, 7001)},
      "S": {"col1": ko, "col2": rng.integers(-50, 50, 50011), "col3": rng.integers(0, 3, 50011)}}
Ro, So = eng.load_table(to["R"], dtypes={"col1": "int64"}), eng.load_table(to["S"], dtypes={"col1": "int64"})
for preds in ([], [{"col": "col3", "op": "!=", "lit": 1}]):
    for agg in ("min", "exists"):
        plan = make_plan("=", agg, "<=", inner_preds=preds)
        g = eng.result_to_numpy(eng.exec(plan, Ro, So, index=eng.index_for_plan(plan, So), emit_all=True))
        ref = oracle.evaluate(to, plan)
        bad += not np.array_equal(g["value"], ref["value"][ref["in_rp"].astype(bool)])
eng.set_option(OPT_SORT, 2)
for keys, dt, pay in ((rng.integers(0, 1 << 27, 100003), "int32", True),
                      (rng.integers(0, 1 << 29, 100003) + (7 << 40), "int64", False),
                      (rng.integers(-2 ** 40, 2 ** 40, 60007), "int64", True)):
    cols = {"k": keys, "v": np.arange(len(keys))} if pay else {"k": keys}
    T = eng.load_table(cols, dtypes={"k": dt, "v": "int32"} if pay else {"k": dt})
    ix = eng.build_index(T, ["k"], "v" if pay else None)
    info = eng.index_info(ix)
    kb = info["key_bytes"]
    got = eng.arena_view(info["d_keys"], len(keys) * kb).view(torch.int64 if kb == 8 else torch.int32).cpu().numpy()
    enc = (keys.astype(np.int64).view(np.uint64) ^ np.uint64(1 << 63)) if kb == 8 else \
        (keys.astype(np.int32).view(np.uint32) ^ np.uint32(1 << 31))
    bad += not np.array_equal(got.view(enc.dtype), np.sort(enc))
eng.set_option(OPT_SORT, 0)
eng.cost_calibrate(1 << 16)
print("sanitize workload done, mismatches:", bad)
sys.exit(1 if bad else 0)
