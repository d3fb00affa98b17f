"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element, on the same seeded inputs.  Integer work -> bit-exact.

Covers both subquery kernels (index path: sort + binary search + range
aggregate; nested-loop path: tiled BNL) for every correlated operator and
aggregate, NULLs and empty subqueries, local predicates, composite keys,
64-bit keys / payloads, extreme values, ragged sizes spanning many tiles,
the BASELINE configs (C1 full; C2 full with sampled oracle rows; C5-shaped),
and the ABI's error paths.
"""
import zlib

import numpy as np
import pytest

import oracle
from datagen import make_plan, PLAN_OPS, query1
from tests import independent as ind
from tests.gpu_helpers import run, assert_parity, make_engine

pytestmark = pytest.mark.gpu

AGGS = ("min", "max", "sum", "count", "avg", "exists", "not_exists")
MODES = ("bnl", "index")


@pytest.fixture(scope="module")
def eng():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    e = make_engine(16)
    yield e
    e.close()


# ------------------------------------------------------------------ C1
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("corr_op", PLAN_OPS)
def test_c1_all_aggs(eng, mode, corr_op):
    t = query1.config("C1")
    for agg in AGGS:
        for outer_op in (("=",) if agg in ("exists", "not_exists") else ("=", "<", ">=")):
            plan = make_plan(corr_op, agg, outer_op)
            ref = oracle.evaluate(t, plan)
            assert_parity(run(eng, t, plan, mode, emit_all=True), ref, plan, True, ctx=(mode, corr_op, agg, outer_op))
            assert_parity(run(eng, t, plan, mode, emit_all=False), ref, plan, False, ctx=(mode, corr_op, agg, outer_op))


# ------------------------------------------------------------------ NULLs, predicates, ragged
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("seed", [1, 2])
def test_nulls_predicates_ragged(eng, mode, seed):
    # |R| = 9001 and |S| = 13007 span several 4096-row filter tiles and
    # 2048-element BNL tiles / R blocks with ragged tails.
    t = query1.random_small(seed, n_r=9001, n_s=13007, key_hi=3000, val_lo=-50, val_hi=50, null_frac=0.1)
    for corr_op in PLAN_OPS:
        for agg in AGGS:
            plan = make_plan(corr_op, agg, PLAN_OPS[(seed + len(agg)) % 6],
                             outer_preds=[{"col": "col3", "op": "<=", "lit": 1}],
                             inner_preds=[{"col": "col3", "op": "!=", "rhs": "col2"}],
                             lhs_mult=2, rhs_mult=3)
            ref = oracle.evaluate(t, plan)
            assert_parity(run(eng, t, plan, mode, emit_all=True), ref, plan, True, ctx=(mode, corr_op, agg))


@pytest.mark.parametrize("mode", MODES)
def test_composite_key(eng, mode):
    t = query1.random_small(5, n_r=7000, n_s=11000, key_hi=40, null_frac=0.05)
    for agg in AGGS:
        plan = make_plan("=", agg, "<=", outer_key=["col1", "col3"], inner_key=["col1", "col3"])
        ref = oracle.evaluate(t, plan)
        assert_parity(run(eng, t, plan, mode, emit_all=True), ref, plan, True, ctx=(mode, agg))


@pytest.mark.parametrize("mode", MODES)
def test_int64_keys_and_payloads(eng, mode):
    rng = np.random.default_rng(8)
    n_r, n_s = 5000, 9000
    keys = rng.integers(-2 ** 40, 2 ** 40, size=600)
    t = {"R": {"k": rng.choice(keys, n_r), "x": rng.integers(-10 ** 12, 10 ** 12, n_r)},
         "S": {"k": rng.choice(keys, n_s), "v": rng.integers(-10 ** 12, 10 ** 12, n_s)}}
    t["R"]["k"][:50] = rng.integers(-2 ** 62, 2 ** 62, 50)  # some keys absent from S
    for corr_op in PLAN_OPS:
        for agg in AGGS:
            plan = make_plan(corr_op, agg, "<", outer_key=["k"], inner_key=["k"], agg_col="v", outer_cmp_col="x")
            ref = oracle.evaluate(t, plan)
            assert_parity(run(eng, t, plan, mode, emit_all=True), ref, plan, True, ctx=(mode, corr_op, agg))


@pytest.mark.parametrize("mode", MODES)
def test_mixed_key_widths(eng, mode):
    # int32 outer key against int64 inner key (and decimals as int64)
    rng = np.random.default_rng(9)
    t = {"R": {"k": rng.integers(-100, 100, 3000).astype(np.int32), "x": rng.integers(0, 300, 3000)},
         "S": {"k": rng.integers(-100, 100, 4000).astype(np.int64), "v": rng.integers(-500, 500, 4000)}}
    for corr_op in ("=", "<", "!="):
        for agg in ("min", "avg", "count"):
            plan = make_plan(corr_op, agg, ">", outer_key=["k"], inner_key=["k"], agg_col="v", outer_cmp_col="x")
            ref = oracle.evaluate(t, plan)
            assert_parity(run(eng, t, plan, mode, emit_all=True,
                              dtypes={"S": {"v": "decimal"}}), ref, plan, True, ctx=(mode, corr_op, agg))


@pytest.mark.parametrize("mode", MODES)
def test_extreme_values(eng, mode):
    # INT32_MIN / INT32_MAX keys and payloads: exercises the order-preserving
    # key encoding and the MIN/MAX identity tracking (payload == identity).
    i32 = np.iinfo(np.int32)
    rng = np.random.default_rng(10)
    dom = np.array([i32.min, i32.min + 1, -1, 0, 1, i32.max - 1, i32.max], np.int32)
    t = {"R": {"col1": rng.choice(dom, 3000), "col2": rng.choice(dom, 3000)},
         "S": {"col1": rng.choice(dom, 5000), "col2": rng.choice(dom, 5000)}}
    for corr_op in PLAN_OPS:
        for agg in AGGS:
            plan = make_plan(corr_op, agg, "=")
            ref = oracle.evaluate(t, plan)
            assert_parity(run(eng, t, plan, mode, emit_all=True), ref, plan, True, ctx=(mode, corr_op, agg))


@pytest.mark.parametrize("mode", MODES)
def test_degenerate(eng, mode):
    e32 = np.zeros(0, np.int32)
    one = np.array([3], np.int32)
    cases = {
        "empty_R": {"R": {"col1": e32, "col2": e32}, "S": {"col1": one, "col2": one}},
        "empty_S": {"R": {"col1": one, "col2": np.array([0], np.int32)}, "S": {"col1": e32, "col2": e32}},
        "single": {"R": {"col1": one, "col2": one}, "S": {"col1": one, "col2": one}},
        "all_null_keys": {"R": {"col1": np.arange(100, dtype=np.int32), "col2": np.zeros(100, np.int32)},
                          "R_valid": {"col1": np.zeros(100, np.uint8)},
                          "S": {"col1": np.arange(50, dtype=np.int32), "col2": np.ones(50, np.int32)}},
    }
    for name, t in cases.items():
        for corr_op in PLAN_OPS:
            for agg in AGGS:
                plan = make_plan(corr_op, agg, "=")
                ref = oracle.evaluate(t, plan)
                assert_parity(run(eng, t, plan, mode, emit_all=True), ref, plan, True, ctx=(name, mode, corr_op, agg))
    # every outer row filtered out / every inner row filtered out
    t = query1.config("C1")
    for preds in ({"outer_preds": [{"col": "col2", "op": "<", "lit": -1}]},
                  {"inner_preds": [{"col": "col2", "op": ">", "lit": 100}]}):
        for agg in AGGS:
            plan = make_plan(">", agg, "=", **preds)
            ref = oracle.evaluate(t, plan)
            assert_parity(run(eng, t, plan, mode, emit_all=True), ref, plan, True, ctx=(preds, agg))


# ------------------------------------------------------------------ caching
@pytest.mark.parametrize("mode", MODES)
def test_dedup_caching(eng, mode):
    """dedup = evaluate each distinct correlated value once and reuse the
    result: identical results to the oracle, and the number of
    evaluations equals the number of distinct R' keys."""
    cases = [("c1", query1.config("C1"), {}),
             ("nulls", query1.random_small(3, n_r=9001, n_s=13007, key_hi=300, val_lo=-50, val_hi=50,
                                           null_frac=0.1), {"outer_preds": [{"col": "col3", "op": "<=", "lit": 1}]}),
             ("zipf", query1.tables(n_r=50000, n_s=40000, key_hi=1 << 12, val_hi=16, seed=5, zipf=1.0), {})]
    for name, t, extra in cases:
        for corr_op in PLAN_OPS:
            for agg in AGGS:
                plan = make_plan(corr_op, agg, "<=", **extra)
                ref = oracle.evaluate(t, plan)
                g = run(eng, t, plan, mode, emit_all=True, dedup=True, with_res=True)
                assert_parity(g, ref, plan, True, ctx=(name, mode, corr_op, agg))
                rp = ref["in_rp"].astype(bool)
                assert g["n_evaluated"] == len(np.unique(t["R"]["col1"][rp]))
    # composite keys
    t = query1.random_small(6, n_r=7000, n_s=9000, key_hi=20, null_frac=0.0)
    for agg in AGGS:
        plan = make_plan("=", agg, ">", outer_key=["col1", "col3"], inner_key=["col1", "col3"])
        ref = oracle.evaluate(t, plan)
        assert_parity(run(eng, t, plan, mode, emit_all=True, dedup=True), ref, plan, True, ctx=("composite", agg))


# ------------------------------------------------------------------ C2-shaped
@pytest.mark.parametrize("zipf", [None, 1.0])
def test_c2_shaped_reduced(eng, zipf):
    """C2's distributions at 60,013 x 60,013: every row checked."""
    t = query1.tables(n_r=60013, n_s=60013, key_hi=1 << 14, val_hi=16, seed=2, zipf=zipf)
    for corr_op, agg in query1.C2_SWEEP:
        plan = make_plan(corr_op, agg, "=")
        ref = oracle.evaluate(t, plan)
        for mode in MODES:
            assert_parity(run(eng, t, plan, mode, emit_all=True), ref, plan, True, ctx=(mode, corr_op, agg, zipf))
            assert_parity(run(eng, t, plan, mode, emit_all=False), ref, plan, False, ctx=(mode, corr_op, agg, zipf))


def test_c2_full_size(eng):
    """BASELINE configs[1] at full size (|R|=|S|=1M), in the bench's launch
    configuration ('=' on the index path, '<', '>', '!=' on the BNL path):
    oracle on 1500 sampled rows, closed-form checker on every row."""
    t = query1.config("C2")
    rng = np.random.default_rng(0)
    rows = np.unique(np.concatenate([[0, len(t["R"]["col1"]) - 1], rng.integers(0, len(t["R"]["col1"]), 1500)]))
    for corr_op, agg in query1.C2_SWEEP:
        plan = make_plan(corr_op, agg, "=")
        mode = "index" if corr_op == "=" else "bnl"
        g = run(eng, t, plan, mode, emit_all=True)
        ref = oracle.evaluate(t, plan, rows=rows)
        assert_parity(g, ref, plan, True, rows=rows, ctx=(corr_op, agg))
        valid, value, cnt, s_sum = ind.closed_form(t["R"]["col1"], t["S"]["col1"], t["S"]["col2"], corr_op, agg)
        assert np.array_equal(g["valid"].astype(bool), valid), (corr_op, agg)
        assert np.array_equal(g["value"], value), (corr_op, agg)
        # the outer comparison on every row (not only the oracle's sample)
        passed = ind.outer_passed(t["R"]["col2"], valid, value, cnt, s_sum, agg, "=")
        assert np.array_equal(g["passed"].astype(bool), passed), (corr_op, agg)
        s = run(eng, t, plan, mode, emit_all=False)
        exp = np.nonzero(g["passed"])[0]
        assert np.array_equal(s["row"], exp)


def test_c5_shaped(eng):
    """C5's distributions (keys U[0,2^31-1), values U[0,2^20)) with |S| = 16M
    and |R| = 131,072: '>' min on the BNL path; oracle on sampled rows plus
    the closed form on every row."""
    t = query1.config("C5", n_r=131072)
    rows = np.unique(np.random.default_rng(1).integers(0, 131072, 300))
    for agg in ("min", "count"):
        plan = make_plan(">", agg, "=")
        g = run(eng, t, plan, "bnl", emit_all=True)
        ref = oracle.evaluate(t, plan, rows=rows)
        assert_parity(g, ref, plan, True, rows=rows, ctx=agg)
        valid, value, _, _ = ind.closed_form(t["R"]["col1"], t["S"]["col1"], t["S"]["col2"], ">", agg)
        assert np.array_equal(g["value"], value)
        assert np.array_equal(g["valid"].astype(bool), valid)


# ------------------------------------------------------------------ index content
def test_index_contents(eng):
    """The index is S' sorted by encoded key with the payload carried along:
    keys ascending, and the (key, payload) multiset equals S's.  (S' rows
    reach the sort in tile-claim order, so the order among equal keys is not
    fixed; no aggregate depends on it.)"""
    import torch
    rng = np.random.default_rng(4)
    n = 300007
    k = rng.integers(-2 ** 31, 2 ** 31, n, dtype=np.int64).astype(np.int32)
    k[::3] = 7  # many duplicates
    v = np.arange(n, dtype=np.int32)
    m = eng.mark()
    try:
        S = eng.load_table({"k": k, "v": v})
        ix = eng.build_index(S, ["k"], "v")
        info = eng.index_info(ix)
        assert info["n"] == n and info["key_bytes"] == 4 and info["payload_bytes"] == 4
        keys = eng.arena_view(info["d_keys"], n * 4).view(torch.int32).cpu().numpy().view(np.uint32)
        pay = eng.arena_view(info["d_payload"], n * 4).view(torch.int32).cpu().numpy()
        enc = k.view(np.uint32) ^ np.uint32(0x80000000)
        assert np.all(keys[1:] >= keys[:-1])
        assert np.array_equal(np.sort(pay), v)              # every payload exactly once
        assert np.array_equal(keys, enc[pay])               # carried with its own key
    finally:
        eng.release(m)


def test_index_prefix_aggregates_survive_release(eng):
    """Index-pruned evaluation (NEXT 3): the prefix / suffix aggregates an
    exec attaches to an index are dropped with a release of a later mark and
    rebuilt on the next use -- results stay exact."""
    t = query1.config("C1")
    m0 = eng.mark()
    try:
        R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
        ix = eng.build_index(S, ["col1"], "col2")
        for agg in ("min", "max", "sum", "avg"):
            plan = make_plan("!=", agg, "<")
            ref = oracle.evaluate(t, plan)
            m1 = eng.mark()
            g1 = eng.result_to_numpy(eng.exec(plan, R, S, index=ix, emit_all=True))
            eng.release(m1)                      # drops the aggregates built after m1
            eng.load_column(np.full(4096, 7, np.int32))   # reuse that arena space
            g2 = eng.result_to_numpy(eng.exec(plan, R, S, index=ix, emit_all=True))
            for g in (g1, g2):
                assert_parity(g, ref, plan, True, ctx=agg)
    finally:
        eng.release(m0)


# ------------------------------------------------------------------ errors
def test_error_paths(eng):
    from paper_conf_icde_floratosxwgylz21_b200 import NestGPUError, Engine
    t = query1.config("C1")
    m = eng.mark()
    try:
        R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
        bad = dict(make_plan("<", "min", "="), outer_key=["col1", "col2"], inner_key=["col1", "col2"])
        with pytest.raises(NestGPUError) as ei:
            eng.exec(bad, R, S)
        assert ei.value.code == -4  # composite non-equality: UNSUPPORTED
        with pytest.raises(NestGPUError) as ei:
            eng.exec(make_plan("=", "min", "=", lhs_mult=0), R, S)
        assert ei.value.code == -1
        ix = eng.build_index(S, ["col1"], "col2")
        with pytest.raises(NestGPUError) as ei:
            eng.exec(make_plan("=", "min", "=", inner_preds=[{"col": "col2", "op": ">", "lit": 3}]), R, S, index=ix)
        assert ei.value.code == -1  # index built with other inner predicates
        res = eng.exec(make_plan("=", "count", "="), R, S, index=ix, emit_all=True)
        import ctypes
        buf = np.empty(1, np.int64)
        st = eng.lib.nestgpu_result_to_host(eng.ctx, ctypes.byref(res), ctypes.c_void_p(buf.ctypes.data),
                                            None, None, None, None, None, 1)
        assert st == -7  # BUFFER
        big = {"k": np.zeros(4, np.int64), "v": np.full(4, 2 ** 62, np.int64)}
        S2 = eng.load_table(big, dtypes={"v": "decimal"})
        R2 = eng.load_table({"k": np.zeros(2, np.int64), "x": np.zeros(2, np.int64)})
        with pytest.raises(NestGPUError) as ei:
            eng.exec(make_plan("=", "sum", "=", outer_key=["k"], inner_key=["k"], agg_col="v", outer_cmp_col="x"), R2, S2)
        assert ei.value.code == -5  # OVERFLOW: the group's exact sum (2^64) leaves int64
    finally:
        eng.release(m)
    small = Engine(0, arena_bytes=1 << 20)
    with pytest.raises(NestGPUError) as ei:
        small.load_column(np.zeros(1 << 20, np.int32))
    assert ei.value.code == -2  # OOM
    small.close()


def test_launch_count_and_profile(eng):
    t = query1.config("C1")
    m = eng.mark()
    try:
        R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
        from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_TINY
        eng.set_profiling(True)
        before = eng.launch_count()
        eng.exec(make_plan(">", "min", "="), R, S)
        assert eng.launch_count() - before == 1   # the one-launch tiny path
        prof = eng.last_profile()
        assert prof["subquery"] > 0 and prof["total"] >= prof["subquery"]
        eng.set_option(OPT_TINY, 0)
        before = eng.launch_count()
        eng.exec(make_plan(">", "min", "="), R, S)
        assert eng.launch_count() - before >= 4  # fill, R' filter, S' filter, BNL, finalize
        prof = eng.last_profile()
        assert prof["subquery"] > 0 and prof["total"] >= prof["subquery"]
    finally:
        eng.set_option(OPT_TINY, 1)
        eng.set_profiling(False)
        eng.release(m)


# ------------------------------------------------------------------ skew extremes
@pytest.mark.parametrize("mode", MODES)
def test_all_keys_equal_and_two_keys(eng, mode):
    """Degenerate key distributions: every S key equal (every radix digit is
    constant -> no sort pass; one '=' range spans all of S -> the long-range
    path) and only two distinct keys (one populated digit)."""
    rng = np.random.default_rng(12)
    for name, sk in (("one_key", np.full(70001, 5, np.int32)),
                     ("two_keys", rng.choice(np.array([5, 1 << 20], np.int32), 70001))):
        t = {"R": {"col1": rng.choice(np.array([4, 5, 6, 1 << 20], np.int32), 5003),
                   "col2": rng.integers(0, 40, 5003).astype(np.int32)},
             "S": {"col1": sk, "col2": rng.integers(-100, 100, 70001).astype(np.int32)}}
        for corr_op in PLAN_OPS:
            for agg in AGGS:
                plan = make_plan(corr_op, agg, ">")
                ref = oracle.evaluate(t, plan)
                for dedup in (False, True):
                    assert_parity(run(eng, t, plan, mode, emit_all=True, dedup=dedup), ref, plan, True,
                                  ctx=(name, mode, corr_op, agg, dedup))


def test_c2_zipf_full_size_cached(eng):
    """C2's Zipf(1.0) variant at full size (1M x 1M) with caching on: the
    index path ('=') and the nested loop ('<', '>', '!='), oracle on sampled
    rows + closed form on every row."""
    t = query1.config("C2z")
    rng = np.random.default_rng(3)
    rows = np.unique(rng.integers(0, 1_000_000, 400))
    for corr_op, agg in query1.C2_SWEEP:
        plan = make_plan(corr_op, agg, "=")
        mode = "index" if corr_op == "=" else "bnl"
        g = run(eng, t, plan, mode, emit_all=True, dedup=True, with_res=True)
        assert g["n_evaluated"] == len(np.unique(t["R"]["col1"]))
        ref = oracle.evaluate(t, plan, rows=rows)
        assert_parity(g, ref, plan, True, rows=rows, ctx=("zipf", corr_op, agg))
        valid, value, _, _ = ind.closed_form(t["R"]["col1"], t["S"]["col1"], t["S"]["col2"], corr_op, agg)
        assert np.array_equal(g["valid"].astype(bool), valid) and np.array_equal(g["value"], value)


# ------------------------------------------------------------------ ablation knob
@pytest.mark.parametrize("mode", MODES)
def test_malloc_scratch_option_same_result(eng, mode):
    """NESTGPU_OPT_MALLOC_SCRATCH (the pool-less ablation baseline)
    changes where scratch lives, never the result."""
    from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_MALLOC_SCRATCH
    t = query1.config("C1")
    for corr_op in ("=", ">", "!="):
        for agg in ("min", "avg", "count"):
            plan = make_plan(corr_op, agg, "=")
            ref = oracle.evaluate(t, plan)
            eng.set_option(OPT_MALLOC_SCRATCH, 1)
            try:
                got = run(eng, t, plan, mode, emit_all=True)
            finally:
                eng.set_option(OPT_MALLOC_SCRATCH, 0)
            assert_parity(got, ref, plan, True, ctx=("malloc", mode, corr_op, agg))


# ------------------------------------------------------------------ both R-block shapes
@pytest.mark.parametrize("shape", ["split", "full"])
def test_bnl_block_shapes_ragged(eng, shape):
    """The nested-loop kernel picks full R blocks (2048 tuples, every warp its
    own) or the warp-split shape (256 tuples shared by 8 warps, each scanning
    1/8 of every S' tile) from the device counts.  Both shapes, ragged R and S
    tails, every operator x aggregate: closed form on every row + the oracle
    on sampled rows."""
    if shape == "split":
        t = query1.tables(n_r=1999, n_s=250_001, key_hi=1 << 16, val_hi=1 << 12, seed=31)
    else:
        t = query1.tables(n_r=40_001, n_s=250_001, key_hi=1 << 16, val_hi=1 << 12, seed=32)
    n_r = len(t["R"]["col1"])
    rows = np.unique(np.random.default_rng(5).integers(0, n_r, 40))
    for corr_op in PLAN_OPS:
        for agg in ("min", "max", "sum", "count", "avg", "exists"):
            plan = make_plan(corr_op, agg, "<")
            g = run(eng, t, plan, "bnl", emit_all=True)
            valid, value, _, _ = ind.closed_form(t["R"]["col1"], t["S"]["col1"], t["S"]["col2"], corr_op, agg)
            assert np.array_equal(g["value"], value), (shape, corr_op, agg)
            assert np.array_equal(g["valid"].astype(bool), valid), (shape, corr_op, agg)
            if corr_op in ("<", "!=") and agg in ("min", "avg"):
                ref = oracle.evaluate(t, plan, rows=rows)
                assert_parity(g, ref, plan, True, rows=rows, ctx=(shape, corr_op, agg))


@pytest.mark.parametrize("shape", [1, 2])
def test_bnl_shape_knob(eng, shape):
    """NESTGPU_OPT_BNL_SHAPE forces full or warp-split R blocks on the same
    input (C1 + NULL-bearing random tables): identical to the oracle."""
    from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_BNL_SHAPE
    tabs = [query1.config("C1"), query1.random_small(17, n_r=3001, n_s=5003, key_hi=500, val_lo=-9, val_hi=9,
                                                      null_frac=0.1)]
    eng.set_option(OPT_BNL_SHAPE, shape)
    try:
        for t in tabs:
            for corr_op in PLAN_OPS:
                for agg in AGGS:
                    plan = make_plan(corr_op, agg, "<=")
                    assert_parity(run(eng, t, plan, "bnl", emit_all=True), oracle.evaluate(t, plan), plan, True,
                                  ctx=(shape, corr_op, agg))
    finally:
        eng.set_option(OPT_BNL_SHAPE, 0)


@pytest.mark.parametrize("base", [0, 5 << 40, -(3 << 40)])
def test_int64_keys_narrowed_sort(eng, base):
    """64-bit keys whose high 32 bits all agree are radix-sorted as 32-bit
    keys between the first and the last pass (the high word re-attached at
    the end): index path and caching (R' key sort), vs the oracle."""
    rng = np.random.default_rng(abs(base) % 97 + 1)
    t = {"R": {"col1": base + rng.integers(0, 1 << 20, 30001), "col2": rng.integers(-40, 40, 30001)},
         "S": {"col1": base + rng.integers(0, 1 << 20, 40003), "col2": rng.integers(-40, 40, 40003)}}
    dt = {"R": {"col1": "int64", "col2": "int64"}, "S": {"col1": "int64", "col2": "int64"}}
    for corr_op in ("=", "<", "!="):
        for agg in ("min", "count"):
            plan = make_plan(corr_op, agg, ">=")
            ref = oracle.evaluate(t, plan)
            for dedup in (False, True):
                g = run(eng, t, plan, "index", emit_all=True, dtypes=dt, dedup=dedup)
                assert_parity(g, ref, plan, True, ctx=(base, corr_op, agg, dedup))


@pytest.mark.parametrize("corr_op,agg", [(">", "min"), (">", "count"), ("!=", "min")])
def test_c5_full_size(eng, corr_op, agg):
    """BASELINE configs[4] at its full size (|R| = |S| = 16M, nested loop --
    bench.py's headline launch configuration, '>' MIN, and its side plans
    '>' COUNT and '!=' MIN, SURVEY §8(d) "Also run count and !="): the closed
    form on every one of the 16M rows (value, valid and the outer comparison
    'passed'), the oracle on 200 sampled rows."""
    t = query1.config("C5")
    plan = make_plan(corr_op, agg, "=")
    rows = np.unique(np.random.default_rng(9).integers(0, 16_000_000, 200))
    g = run(eng, t, plan, "bnl", emit_all=True)
    valid, value, cnt, s_sum = ind.closed_form(t["R"]["col1"], t["S"]["col1"], t["S"]["col2"], corr_op, agg)
    assert np.array_equal(g["value"], value)
    assert np.array_equal(g["valid"].astype(bool), valid)
    passed = ind.outer_passed(t["R"]["col2"], valid, value, cnt, s_sum, agg, "=")
    assert np.array_equal(g["passed"].astype(bool), passed)
    assert_parity(g, oracle.evaluate(t, plan, rows=rows), plan, True, rows=rows, ctx=("C5 full", corr_op, agg))


def _key_pattern(name, n, rng):
    """Encoded-key bit patterns for the radix-pass planner (api.cpp
    plan_sort_passes): which bits vary decides where the 8-bit windows go."""
    if name == "mult32_lt2^26":       # varying bits 5..25 -> 3 windows (5, 13, 21)
        return rng.integers(0, 1 << 21, n) * 32, "int32"
    if name == "bits1_to_27":         # 27 varying bits from bit 1 -> windows 1, 9, 17, 24 (clamped)
        return rng.integers(0, 1 << 27, n) * 2, "int32"
    if name == "i64_low_word":        # 64-bit, high word constant, bits 3..31 vary (narrowed passes, clamp)
        return (7 << 40) + rng.integers(0, 1 << 29, n) * 8, "int64"
    if name == "i64_straddle":        # 64-bit, bits 20..44 vary (windows cross bit 32, no narrowing)
        return -(1 << 50) + rng.integers(0, 1 << 25, n) * (1 << 20), "int64"
    if name == "i64_full":            # all 64 bits vary
        return rng.integers(-2 ** 63, 2 ** 63 - 1, n, dtype=np.int64), "int64"
    if name == "i64_all_equal":       # 64-bit, one value: no bit varies (the narrowed filter output still widens)
        return np.full(n, (7 << 40) + 3, dtype=np.int64), "int64"
    if name == "i32_negative_dups":   # signed, heavy duplicates
        k = rng.integers(-1000, 1000, n)
        k[::5] = -7
        return k, "int32"
    raise KeyError(name)


@pytest.mark.parametrize("pattern", ["mult32_lt2^26", "bits1_to_27", "i64_low_word", "i64_straddle",
                                     "i64_full", "i64_all_equal", "i32_negative_dups"])
@pytest.mark.parametrize("n", [1, 2, 4095, 4097, 1_000_003])
@pytest.mark.parametrize("pay", ["int32", "int64", None])
def test_index_sort_digit_windows(eng, pattern, n, pay):
    """a4 on key patterns whose varying bits sit at odd offsets, cross bit 32,
    or span all 64 bits; 4/8-byte payloads or none (8- to 16-byte items, two
    tile sizes); sizes below, at and across tile boundaries.  The index must
    be the encoded keys ascending with every payload carried by its own key
    (compared with numpy's sort of the same encoded keys)."""
    import torch
    rng = np.random.default_rng([zlib.crc32(pattern.encode()), n])   # deterministic (str hash is salted)
    k, kdt = _key_pattern(pattern, n, rng)
    k = np.asarray(k, dtype=np.int64)
    cols, dts = {"k": k}, {"k": kdt}
    if pay is not None:
        cols["v"] = np.arange(n, dtype=np.int64) * (1 if pay == "int32" else (1 << 33) + 1)
        dts["v"] = pay
    m = eng.mark()
    try:
        S = eng.load_table(cols, dtypes=dts)
        ix = eng.build_index(S, ["k"], "v" if pay else None)
        info = eng.index_info(ix)
        kb = 4 if kdt == "int32" else 8
        assert info["n"] == n and info["key_bytes"] == kb
        if kb == 4:
            enc = k.astype(np.int32).view(np.uint32) ^ np.uint32(0x80000000)
            keys = eng.arena_view(info["d_keys"], n * 4).view(torch.int32).cpu().numpy().view(np.uint32)
        else:
            enc = k.view(np.uint64) ^ np.uint64(1 << 63)
            keys = eng.arena_view(info["d_keys"], n * 8).view(torch.int64).cpu().numpy().view(np.uint64)
        assert np.array_equal(keys, np.sort(enc))
        if pay is not None:
            vb = 4 if pay == "int32" else 8
            tdt = torch.int32 if vb == 4 else torch.int64
            p = eng.arena_view(info["d_payload"], n * vb).view(tdt).cpu().numpy().astype(np.int64)
            row = p if vb == 4 else p // ((1 << 33) + 1)
            assert np.array_equal(np.sort(row), np.arange(n))       # every payload exactly once
            assert np.array_equal(keys, enc[row])                   # carried with its own key
    finally:
        eng.release(m)


@pytest.mark.parametrize("pattern", ["bits1_to_27", "i64_low_word", "i32_negative_dups"])
@pytest.mark.parametrize("pay", ["int32", "int64"])
def test_index_sort_large(eng, pattern, pay):
    """3M keys: ~500-1000 tiles in flight across the persistent grid (deep
    look-back walks)."""
    test_index_sort_digit_windows(eng, pattern, 3_000_017, pay)


def _check_index_sorted(eng, ix, k, kdt, pay):
    """The index is the encoded keys ascending, every payload exactly once and
    carried by its own key (payload = row id, scaled for int64)."""
    import torch
    n = len(k)
    info = eng.index_info(ix)
    kb = 4 if kdt == "int32" else 8
    assert info["n"] == n and info["key_bytes"] == kb
    if kb == 4:
        enc = k.astype(np.int32).view(np.uint32) ^ np.uint32(0x80000000)
        keys = eng.arena_view(info["d_keys"], n * 4).view(torch.int32).cpu().numpy().view(np.uint32)
    else:
        enc = k.view(np.uint64) ^ np.uint64(1 << 63)
        keys = eng.arena_view(info["d_keys"], n * 8).view(torch.int64).cpu().numpy().view(np.uint64)
    assert np.array_equal(keys, np.sort(enc))
    if pay is not None:
        vb = 4 if pay == "int32" else 8
        tdt = torch.int32 if vb == 4 else torch.int64
        p = eng.arena_view(info["d_payload"], n * vb).view(tdt).cpu().numpy().astype(np.int64)
        row = p if vb == 4 else p // ((1 << 33) + 1)
        assert np.array_equal(np.sort(row), np.arange(n))
        assert np.array_equal(keys, enc[row])
        return keys, row
    return keys, None


@pytest.mark.parametrize("kdt", ["int32", "int64"])
@pytest.mark.parametrize("pay", ["int32", "int64", None])
@pytest.mark.parametrize("n,pred", [(1, False), (5000, False), (300_007, True), (2_000_003, True),
                                    (2_000_003, False)])
def test_index_key_ordered_column(eng, kdt, pay, n, pred):
    """Sort-free index build: a NOT NULL key column stored in ascending order
    (column statistics; TPC-H lineitem by l_orderkey, partsupp by ps_partkey)
    is compacted in row order by the ordered filter straight into the index.
    The stable sort of S' is the identity, so the index must be S' exactly:
    keys ascending and, within equal keys, payloads in row order -- and the
    LSD sort of the same S (NESTGPU_OPT_SORT = 1) must hold the same keys and
    the same (key, payload) pairs.  Then '=' / '<' plans through both indexes
    vs the oracle."""
    from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_SORT
    import torch
    rng = np.random.default_rng([n, len(kdt), 0 if pay is None else len(pay)])
    k = np.sort(rng.integers(-(1 << 33) if kdt == "int64" else -(1 << 20), 1 << 20, n))
    k[n // 3: n // 3 + min(n, 50)] = k[n // 3] if n > 1 else k[:1]   # a long run of one key
    k = np.sort(k)
    v = rng.integers(-1000, 1000, n) * (1 if pay != "int64" else (1 << 34))
    c3 = rng.integers(0, 4, n)
    cols, dts = {"col1": k, "col3": c3}, {"col1": kdt, "col3": "int32"}
    if pay is not None:
        cols["col2"], dts["col2"] = v, pay
    preds = [{"col": "col3", "op": "!=", "lit": 1}] if pred else []
    keep = c3 != 1 if pred else np.ones(n, bool)
    m = eng.mark()
    try:
        S = eng.load_table(cols, dtypes=dts)
        got = {}
        for mode in (0, 1):
            eng.set_option(OPT_SORT, mode)
            eng.set_profiling(True)
            ix = eng.build_index(S, ["col1"], "col2" if pay else None, preds)
            prof = eng.last_profile()
            eng.set_profiling(False)
            info = eng.index_info(ix)
            ns = int(keep.sum())
            assert info["n"] == ns
            kb = 4 if kdt == "int32" else 8
            tdt = torch.int32 if kb == 4 else torch.int64
            keys = np.zeros(0, np.int64)
            if ns:
                kr = eng.arena_view(info["d_keys"], ns * kb).view(tdt).cpu().numpy()
                keys = kr.view(np.uint32).astype(np.int64) if kb == 4 else kr
            enc = k[keep].astype(np.int64)
            enc_u = (enc.astype(np.int32).view(np.uint32) ^ np.uint32(1 << 31)).astype(np.int64) if kb == 4 else \
                (enc.view(np.uint64) ^ np.uint64(1 << 63)).view(np.int64)
            assert np.array_equal(keys, enc_u)
            p = None
            if pay is not None and ns:
                vbt = torch.int32 if pay == "int32" else torch.int64
                vbb = 4 if pay == "int32" else 8
                p = eng.arena_view(info["d_payload"], ns * vbb).view(vbt).cpu().numpy().astype(np.int64)
            got[mode] = (keys, p, prof)
            if mode == 0:
                if pay is not None and ns:
                    assert np.array_equal(p, v[keep])          # row order inside every key run
                assert np.isnan(prof["sort"])                   # no sort ran
        if pay is not None and info["n"]:
            a = np.lexsort((got[0][1], got[0][0]))
            b = np.lexsort((got[1][1], got[1][0]))
            assert np.array_equal(got[0][0][a], got[1][0][b]) and np.array_equal(got[0][1][a], got[1][1][b])
        eng.set_option(OPT_SORT, 0)
        R = {"col1": rng.integers(int(k.min()) - 2, int(k.max()) + 3, 2001), "col2": rng.integers(-1000, 1000, 2001)}
        t = {"R": R, "S": cols}
        dt = {"R": {"col1": kdt, "col2": pay or "int32"}, "S": dts}
        for corr_op, agg in (("=", "min" if pay else "count"), ("=", "exists"), ("<", "count"), ("=", "sum" if pay else "count")):
            plan = make_plan(corr_op, agg, "<=", inner_preds=preds)
            if pay is None and agg in ("min", "sum"):
                continue
            assert_parity(run(eng, t, plan, "index", emit_all=True, dtypes=dt), oracle.evaluate(t, plan), plan, True,
                          ctx=(kdt, pay, n, pred, corr_op, agg))
    finally:
        eng.set_option(OPT_SORT, 0)
        eng.set_profiling(False)
        eng.release(m)


def test_index_almost_ordered_column_sorts(eng):
    """One descent in an otherwise ascending column: not key-ordered, the
    index is sorted (LSD) and still exact; and a caller-filled column whose
    contents change between builds has its order re-checked."""
    import torch
    n = 100_003
    k = np.arange(n, dtype=np.int32) * 3
    k[n // 2], k[n // 2 + 1] = k[n // 2 + 1], k[n // 2]
    m = eng.mark()
    try:
        S = eng.load_table({"col1": k, "col2": np.arange(n, dtype=np.int32)})
        assert eng.index_info(eng.build_index(S, ["col1"], "col2"))["key_bytes"] == 4
        ix = eng.build_index(S, ["col1"], "col2")
        info = eng.index_info(ix)
        keys = eng.arena_view(info["d_keys"], n * 4).view(torch.int32).cpu().numpy().view(np.uint32)
        assert np.array_equal(keys, np.sort(k.astype(np.int32).view(np.uint32) ^ np.uint32(1 << 31)))
        # caller-filled column: first ordered, then rewritten unordered
        cid = eng.alloc_column(n, "int32")
        view = eng.arena_view(eng.column_info(cid)["d_values"], n * 4).view(torch.int32)
        view.copy_(torch.from_numpy(np.arange(n, dtype=np.int32)))
        S2 = dict(S)
        S2["col1"] = cid
        ix2 = eng.build_index(S2, ["col1"], "col2")
        i2 = eng.index_info(ix2)
        got = eng.arena_view(i2["d_keys"], n * 4).view(torch.int32).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), np.arange(n, dtype=np.uint32) ^ np.uint32(1 << 31))
        view.copy_(torch.from_numpy(np.arange(n, dtype=np.int32)[::-1].copy()))
        ix3 = eng.build_index(S2, ["col1"], "col2")
        i3 = eng.index_info(ix3)
        got = eng.arena_view(i3["d_keys"], n * 4).view(torch.int32).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), np.arange(n, dtype=np.uint32) ^ np.uint32(1 << 31))
        pay = eng.arena_view(i3["d_payload"], n * 4).view(torch.int32).cpu().numpy()
        assert np.array_equal(pay, np.arange(n)[::-1])
    finally:
        eng.release(m)


@pytest.mark.parametrize("agg", ["exists", "not_exists", "min", "count"])
def test_result_to_host_survivor_fields(eng, agg):
    """result_to_host writes a survivors-only result's valid / passed (and an
    EXISTS / NOT EXISTS value) on the host instead of copying them: they
    must equal the device fields, on a result too large for the exec's
    pinned staging (C2 '=' plans: 60k-980k survivors)."""
    t = query1.config("C2")
    plan = make_plan("=", agg, "=")
    m = eng.mark()
    try:
        from tests.gpu_helpers import load
        R, S = load(eng, t)
        idx = eng.index_for_plan(plan, S)
        res = eng.exec(plan, R, S, index=idx)
        host = eng.result_to_numpy(res)
        dev = eng.result_tensors(res)
        assert res.n_rows > 20000
        for k in ("row", "value", "valid", "passed"):
            assert np.array_equal(host[k].astype(np.int64), dev[k].cpu().numpy().astype(np.int64)), (agg, k)
        assert host["valid"].all() and host["passed"].all()
    finally:
        eng.release(m)


def _skewed_keys(n, rng):
    """27 varying bits, but 3/4 of the keys in one 2^12-wide range: one
    partition bucket far past the finish capacity (falls back to the LSD
    sort)."""
    k = rng.integers(0, 1 << 27, n)
    k[: 3 * n // 4] = (5 << 20) + rng.integers(0, 1 << 12, 3 * n // 4)
    return rng.permutation(k), "int32"


@pytest.mark.parametrize("pattern", ["mult32_lt2^26", "bits1_to_27", "i64_low_word", "i64_straddle",
                                     "i64_full", "i64_all_equal", "i32_negative_dups", "skewed"])
@pytest.mark.parametrize("n", [2, 4097, 100_003, 1_000_003])
@pytest.mark.parametrize("pay", ["int32", "int64", None])
def test_index_bucket_sort(eng, pattern, n, pay):
    """The two-round-trip MSD bucket sort (k_bsort.cu; NESTGPU_OPT_SORT = 2
    forces it wherever the keys vary in more bits than its partition digit):
    every key pattern, 0/4/8-byte payloads (4- to 16-byte items: every tile /
    bucket register shape), sizes inside one tile, across tiles and groups
    with ragged tails.  Same checks as the LSD sort (which runs beside it on
    the same S)."""
    from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_SORT
    import torch
    rng = np.random.default_rng([zlib.crc32(pattern.encode()), n, 3])
    k, kdt = _skewed_keys(n, rng) if pattern == "skewed" else _key_pattern(pattern, n, rng)
    k = np.asarray(k, dtype=np.int64)
    cols, dts = {"k": k}, {"k": kdt}
    if pay is not None:
        cols["v"] = np.arange(n, dtype=np.int64) * (1 if pay == "int32" else (1 << 33) + 1)
        dts["v"] = pay
    m = eng.mark()
    try:
        S = eng.load_table(cols, dtypes=dts)
        for mode in (2, 1):
            eng.set_option(OPT_SORT, mode)
            ix = eng.build_index(S, ["k"], "v" if pay else None)
            _check_index_sorted(eng, ix, k, kdt, pay)
    finally:
        eng.set_option(OPT_SORT, 0)
        eng.release(m)


@pytest.mark.parametrize("pattern,pay", [("bits1_to_27", "int32"), ("i64_low_word", None),
                                         ("i64_straddle", "int64"), ("skewed", "int32")])
def test_index_bucket_sort_large(eng, pattern, pay):
    """The bucket sort at 3M keys: ~90-370 partition groups, 4096 buckets (the
    skewed keys fall back to the LSD sort after the bucket histogram)."""
    from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_SORT
    eng.set_option(OPT_SORT, 2)
    rng = np.random.default_rng([zlib.crc32(pattern.encode()), 7])
    n = 3_000_017
    k, kdt = _skewed_keys(n, rng) if pattern == "skewed" else _key_pattern(pattern, n, rng)
    k = np.asarray(k, dtype=np.int64)
    cols, dts = {"k": k}, {"k": kdt}
    if pay is not None:
        cols["v"] = np.arange(n, dtype=np.int64) * (1 if pay == "int32" else (1 << 33) + 1)
        dts["v"] = pay
    m = eng.mark()
    try:
        S = eng.load_table(cols, dtypes=dts)
        ix = eng.build_index(S, ["k"], "v" if pay else None)
        _check_index_sorted(eng, ix, k, kdt, pay)
    finally:
        eng.set_option(OPT_SORT, 0)
        eng.release(m)


@pytest.mark.parametrize("pattern", ["mult32_lt2^26", "bits1_to_27", "i64_low_word", "i64_straddle"])
def test_dedup_sort_digit_windows(eng, pattern):
    """The R' key sort of caching on the same key patterns: results
    vs the oracle with and without caching, both subquery kernels."""
    rng = np.random.default_rng(11)
    kr, kdt = _key_pattern(pattern, 20011, rng)
    ks, _ = _key_pattern(pattern, 9001, rng)
    kr = np.asarray(kr, dtype=np.int64)
    rep = np.arange(0, len(kr), 3)
    kr[rep] = kr[(rep + 1) % len(kr)]              # repeated correlated values
    ks = np.concatenate([np.asarray(ks, dtype=np.int64), kr[:3000]])
    t = {"R": {"col1": kr, "col2": rng.integers(0, 5, len(kr))},
         "S": {"col1": ks, "col2": rng.integers(0, 5, len(ks))}}
    dt = {"R": {"col1": kdt, "col2": "int32"}, "S": {"col1": kdt, "col2": "int32"}}
    for corr_op, agg, mode in (("=", "count", "index"), ("=", "min", "index"), ("<", "min", "bnl")):
        plan = make_plan(corr_op, agg, "<=")
        ref = oracle.evaluate(t, plan)
        for dedup in (False, True):
            g = run(eng, t, plan, mode, emit_all=True, dtypes=dt, dedup=dedup)
            assert_parity(g, ref, plan, True, ctx=(pattern, corr_op, agg, dedup))


def test_result_to_numpy_into_buffers(eng):
    """result_to_numpy(out=): the copy into caller buffers (pinned in the
    bench) equals the allocating copy; a buffer that is too small is refused."""
    import torch
    t = query1.config("C1")
    m = eng.mark()
    try:
        R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
        plan = make_plan("=", "avg", "<=")
        res = eng.exec(plan, R, S, index=eng.index_for_plan(plan, S), emit_all=True)
        ref = eng.result_to_numpy(res)
        bufs = {k: torch.empty(2000, dtype=dt, pin_memory=True).numpy()
                for k, dt in (("row", torch.int64), ("value", torch.int64), ("valid", torch.uint8),
                              ("passed", torch.uint8), ("sum", torch.int64), ("cnt", torch.int64))}
        got = eng.result_to_numpy(res, out=bufs)
        assert set(got) == set(ref)
        for k in ref:
            assert np.array_equal(got[k], ref[k]), k
        small = {k: v[:10] for k, v in bufs.items()}
        with pytest.raises(ValueError):
            eng.result_to_numpy(res, out=small)
    finally:
        eng.release(m)


@pytest.mark.parametrize("mode", MODES)
def test_avg_large_int64_payloads(eng, mode):
    """AVG's scaled-integer division (round_half_away(sum * 10^6 / count),
    reading R6) on int64 payloads up to ~9.2e12 in magnitude -- quotients
    near the 64-bit limit and negative sums -- both kernels, vs the oracle."""
    rng = np.random.default_rng(21)
    lim = 9_000_000_000_000
    t = {"R": {"col1": rng.integers(0, 40, 4000), "col2": rng.integers(-lim, lim, 4000)},
         "S": {"col1": rng.integers(0, 40, 6001), "col2": rng.integers(-lim, lim, 6001)}}
    t["S"]["col2"][::7] = lim                      # skewed groups: large positive / negative means
    t["S"]["col2"][1::11] = -lim
    dt = {"R": {"col1": "int32", "col2": "int64"}, "S": {"col1": "int32", "col2": "int64"}}
    for corr_op in ("=", "<", "!="):
        for outer in ("<", ">="):
            plan = make_plan(corr_op, "avg", outer)
            ref = oracle.evaluate(t, plan)
            g = run(eng, t, plan, mode, emit_all=True, dtypes=dt)
            assert_parity(g, ref, plan, True, ctx=(mode, corr_op, outer))


@pytest.mark.parametrize("mode", MODES)
def test_exact_int64_sums_not_refused(eng, mode):
    """SUM/AVG over 64-bit payloads where |S| * max|payload| >= 2^63 but every
    qualifying set's sum fits int64 (pairs (A + x, -A + y) share a key, so
    every '=' group and every key prefix / suffix holds whole pairs): the
    engine must return the oracle's exact values, not NESTGPU_ERR_OVERFLOW
    (reading R5: only a sum that actually leaves int64 is an error).  S rows
    are shuffled, so unit / tile partial sums of the nested loop are random
    walks of +-A that a plain int64 accumulator would wrap."""
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
    for corr_op in PLAN_OPS:
        for agg, outer in (("sum", "<"), ("avg", ">=")):
            plan = make_plan(corr_op, agg, outer)
            ref = oracle.evaluate(t, plan)
            assert_parity(run(eng, t, plan, mode, emit_all=True, dtypes=dt), ref, plan, True,
                          ctx=("wide", mode, corr_op, agg))
    # a real overflow (a qualifying set whose sum leaves int64) is still an
    # error, on both paths, like the oracle's
    from paper_conf_icde_floratosxwgylz21_b200 import NestGPUError
    t2 = {"R": {"col1": np.array([10], np.int64), "col2": np.zeros(1, np.int64)},
          "S": {"col1": np.arange(4, dtype=np.int64), "col2": np.full(4, A, np.int64)}}
    plan = make_plan(">", "sum", "=")
    with pytest.raises(oracle.OracleOverflow):
        oracle.evaluate(t2, plan)
    with pytest.raises(NestGPUError) as ei:
        run(eng, t2, plan, mode, emit_all=True, dtypes=dt)
    assert ei.value.code == -5


def test_c2_zipf_full_size_index_no_cache(eng):
    """C2's Zipf(1.0) variant at full size WITHOUT caching, every aggregate on
    the index path: '=' MIN/MAX read the per-key group aggregates (O(1) per
    outer tuple, no hot-key blow-up), the other operators the prefix /
    suffix aggregates.  Closed form + outer comparison on every row, oracle
    on sampled rows; the '=' MIN kernel must stay far below the per-tuple
    fold of the hot keys' runs (sum over keys of |R_k| x |S_k|, ~1e10
    element visits)."""
    import time
    t = query1.config("C2z")
    rng = np.random.default_rng(4)
    rows = np.unique(rng.integers(0, 1_000_000, 300))
    for corr_op in ("=", "!=", ">"):
        for agg in ("min", "max", "sum", "count"):
            plan = make_plan(corr_op, agg, "=")
            t0 = time.perf_counter()
            g = run(eng, t, plan, "index", emit_all=True)
            dt = time.perf_counter() - t0
            valid, value, cnt, s_sum = ind.closed_form(t["R"]["col1"], t["S"]["col1"], t["S"]["col2"], corr_op, agg)
            assert np.array_equal(g["valid"].astype(bool), valid), (corr_op, agg)
            assert np.array_equal(g["value"], value), (corr_op, agg)
            passed = ind.outer_passed(t["R"]["col2"], valid, value, cnt, s_sum, agg, "=")
            assert np.array_equal(g["passed"].astype(bool), passed), (corr_op, agg)
            ref = oracle.evaluate(t, plan, rows=rows)
            assert_parity(g, ref, plan, True, rows=rows, ctx=("zipf nocache", corr_op, agg))
            assert dt < 5.0, (corr_op, agg, dt)   # load + index + exec + copy-out


def test_exec_graph_replay_matches(eng):
    """NESTGPU_OPT_GRAPHS: the exec launch sequence is captured into a CUDA
    graph on first use and replayed afterwards.  Replays give the oracle's
    result on every call, identical to running with graphs off, including
    after the column contents change in place (a graph references addresses,
    not data) and for the split-SUM path."""
    import torch
    from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_GRAPHS
    t = query1.random_small(7, n_r=3001, n_s=4001, key_hi=50, val_lo=-9, val_hi=9, null_frac=0.1)
    plans = [(make_plan(op, agg, "<", outer_preds=[{"col": "col3", "op": "<=", "lit": 1}]), mode)
             for op, agg, mode in (("=", "min", "index"), (">", "count", "bnl"), ("!=", "sum", "bnl"),
                                   ("<", "avg", "index"), ("=", "exists", "bnl"))]
    m = eng.mark()
    try:
        R = eng.load_table(t["R"], t.get("R_valid"))
        S = eng.load_table(t["S"], t.get("S_valid"))
        for graphs in (1, 0, 1):
            eng.set_option(OPT_GRAPHS, graphs)
            for plan, mode in plans:
                ref = oracle.evaluate(t, plan)
                idx = eng.index_for_plan(plan, S) if mode == "index" else -1
                for rep in range(11):   # 8 direct runs, the capture, replays
                    g = eng.result_to_numpy(eng.exec(plan, R, S, index=idx, emit_all=True))
                    assert_parity(g, ref, plan, True, ctx=("graphs", graphs, plan["corr_op"], plan["agg"], rep))
                    # survivors only: the cooperative compaction kernel inside the graph
                    g = eng.result_to_numpy(eng.exec(plan, R, S, index=idx, emit_all=False))
                    assert_parity(g, ref, plan, False, ctx=("graphs survivors", graphs, plan["corr_op"], rep))
        # in-place change of R.col2 (the compared column): replays read the new values
        eng.set_option(OPT_GRAPHS, 1)
        plan, mode = plans[1]
        for _ in range(10):
            eng.result_to_numpy(eng.exec(plan, R, S, emit_all=True))
        info = eng.column_info(R["col2"])
        new = (t["R"]["col2"].astype(np.int32) * 3 + 1).astype(np.int32)
        eng.arena_view(info["d_values"], 4 * len(new)).copy_(torch.from_numpy(new.view(np.uint8)))
        t2 = {"R": dict(t["R"], col2=new), "S": t["S"], "R_valid": t["R_valid"], "S_valid": t["S_valid"]}
        g = eng.result_to_numpy(eng.exec(plan, R, S, emit_all=True))
        assert_parity(g, oracle.evaluate(t2, plan), plan, True, ctx="in-place change")
    finally:
        eng.set_option(OPT_GRAPHS, 1)
        eng.release(m)


def test_two_contexts_two_host_threads():
    """Two contexts in one process driven by two host threads at once (the
    ADVICE r1 case: the per-kernel launch setup -- shared-memory opt-ins of
    the nested loop, filter and sort kernels, occupancy -- is cached per
    (kernel, device) under a mutex, not in a process-global static): every
    plan of each thread matches the oracle.  One GPU on this box, so both
    contexts share device 0; each has its own arena and stream."""
    import threading
    from tests.gpu_helpers import make_engine
    t = query1.config("C1")
    plans = [make_plan(op, agg, "=") for op in ("=", ">", "!=") for agg in ("min", "count", "exists")]
    refs = [oracle.evaluate(t, p) for p in plans]
    errors = []

    def work(k):
        try:
            e = make_engine(1)
            try:
                for rep in range(3):
                    for i, p in enumerate(plans):
                        mode = "index" if (i + k + rep) % 2 == 0 else "bnl"
                        assert_parity(run(e, t, p, mode, emit_all=True), refs[i], p, True, ctx=(k, rep, i, mode))
            finally:
                e.close()
        except Exception as ex:   # surfaced below
            errors.append(repr(ex))

    th = [threading.Thread(target=work, args=(k,)) for k in range(2)]
    for x in th:
        x.start()
    for x in th:
        x.join()
    assert not errors, errors


@pytest.mark.parametrize("tiny", [1, 0])
def test_tiny_one_launch_path(eng, tiny):
    """The one-launch path for tiny nested-loop queries (NESTGPU_OPT_TINY,
    k_finalize.cu tiny_exec_kernel) against the oracle and with it switched
    off (the regular fill / filter / nested loop / finalize sequence):
    NULL-bearing random tables with outer and inner predicates (literal and
    column-vs-column), every operator x aggregate x emit mode, a row-id base,
    64-bit keys and decimal payloads, composite keys, and the SUM overflow
    error; sizes at the path's limits (4096 rows, 2^21 pairs)."""
    from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_TINY, NestGPUError
    eng.set_option(OPT_TINY, tiny)
    try:
        t = query1.random_small(23, n_r=511, n_s=4096, key_hi=60, val_lo=-40, val_hi=40, null_frac=0.15)
        for corr_op in PLAN_OPS:
            for agg in AGGS:
                for emit_all in (True, False):
                    plan = make_plan(corr_op, agg, "<=", outer_preds=[{"col": "col3", "op": "<=", "lit": 1}],
                                     inner_preds=[{"col": "col3", "op": "!=", "rhs": "col2"}])
                    ref = oracle.evaluate(t, plan)
                    g = run(eng, t, plan, "bnl", emit_all=emit_all, row_id_base=1000)
                    g["row"] = g["row"] - 1000
                    assert_parity(g, ref, plan, emit_all, ctx=(tiny, corr_op, agg, emit_all))
        rng = np.random.default_rng(5)
        t64 = {"R": {"col1": rng.integers(-3, 40, 4096) * (1 << 35), "col2": rng.integers(-9, 9, 4096) * 10 ** 9},
               "S": {"col1": rng.integers(-3, 40, 512) * (1 << 35), "col2": rng.integers(-9, 9, 512) * 10 ** 12}}
        dt = {"R": {"col1": "int64", "col2": "int64"}, "S": {"col1": "int64", "col2": "decimal"}}
        for corr_op in ("=", "<", "!="):
            for agg in ("min", "sum", "avg", "count"):
                plan = make_plan(corr_op, agg, ">", lhs_mult=1000, rhs_mult=1)
                assert_parity(run(eng, t64, plan, "bnl", emit_all=True, dtypes=dt), oracle.evaluate(t64, plan), plan,
                              True, ctx=(tiny, "i64", corr_op, agg))
        i32 = lambda lo, hi, n: rng.integers(lo, hi, n).astype(np.int32)   # noqa: E731
        tc = {"R": {"a": i32(0, 5, 1500), "b": i32(0, 5, 1500), "x": i32(-5, 5, 1500)},
              "S": {"a": i32(0, 5, 1300), "b": i32(0, 5, 1300), "v": i32(-5, 5, 1300)}}
        for agg in ("max", "count", "not_exists"):
            plan = make_plan("=", agg, "<", outer_key=["a", "b"], inner_key=["a", "b"], agg_col="v", outer_cmp_col="x")
            assert_parity(run(eng, tc, plan, "bnl", emit_all=False), oracle.evaluate(tc, plan), plan, False,
                          ctx=(tiny, "composite", agg))
        big = (1 << 62) + (1 << 61)
        tov = {"R": {"col1": np.zeros(3, np.int64), "col2": np.zeros(3, np.int64)},
               "S": {"col1": np.zeros(4, np.int64), "col2": np.full(4, big, np.int64)}}
        with pytest.raises(NestGPUError):
            run(eng, tov, make_plan("=", "sum", "<"), "bnl", dtypes={"R": {"col1": "int64", "col2": "int64"},
                                                                  "S": {"col1": "int64", "col2": "int64"}})
    finally:
        eng.set_option(OPT_TINY, 1)


@pytest.mark.parametrize("spread", ["dense", "sparse"])
def test_key_ordered_outer_index_path(eng, spread):
    """Ascending outer keys (TPC-H orders by o_orderkey) through the index
    path: every operator x aggregate vs the oracle, ragged warps, duplicate
    outer keys, keys below / above S's range, dense and sparse key spreads."""
    rng = np.random.default_rng(31 if spread == "dense" else 32)
    n_s = 200_003
    s_keys = rng.integers(0, 50_000 if spread == "dense" else 5_000_000, n_s)
    n_r = 40_013
    r_keys = np.sort(rng.integers(-100, (50_000 if spread == "dense" else 5_000_000) + 100, n_r))
    t = {"R": {"col1": r_keys.astype(np.int32), "col2": rng.integers(-60, 60, n_r).astype(np.int32)},
         "S": {"col1": s_keys.astype(np.int32), "col2": rng.integers(-60, 60, n_s).astype(np.int32)}}
    for corr_op in PLAN_OPS:
        for agg in ("min", "count", "sum", "exists"):
            plan = make_plan(corr_op, agg, "<=")
            assert_parity(run(eng, t, plan, "index", emit_all=True), oracle.evaluate(t, plan), plan, True,
                          ctx=(spread, corr_op, agg))
