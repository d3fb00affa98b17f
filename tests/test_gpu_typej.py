"""GPU parity for type-J subqueries and joins with subqueries (PAPER.md
P:197-231): the two-level result arrays
(nestgpu_exec_collect) against the oracle's literal nested loop
(oracle.collect), IN over them (nestgpu_collection_in) against oracle.in_list
and SQLite's literal IN, column materialisation, and the two join-with-
subquery cases of Fig. 5 against SQLite running the SQL directly.

Lists are compared as multisets (the engine emits them in index order, the
oracle in S row order; reading R17).  Everything is integer ->
bit-exact.
"""
import sqlite3

import numpy as np
import pytest

import oracle
from datagen import make_plan, PLAN_OPS, query1
from paper_conf_icde_floratosxwgylz21_b200 import nested
from paper_conf_icde_floratosxwgylz21_b200.binding import NestGPUError, ERR_OVERFLOW, ERR_UNSUPPORTED, ERR_INVALID
from tests import independent as ind
from tests.gpu_helpers import load, make_engine

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def eng():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    e = make_engine(8)
    yield e
    e.close()


def gpu_collect(eng, t, plan, dtypes=None, row_id_base=0):
    m = eng.mark()
    try:
        R, S = load(eng, t, dtypes)
        idx = eng.build_index(S, plan["inner_key"], payload=plan["agg_col"], inner_preds=plan["inner_preds"])
        coll = eng.exec_collect(plan, R, S, idx, row_id_base=row_id_base)
        return eng.collection_to_numpy(coll)
    finally:
        eng.release(m)


def assert_collect_parity(g, ref, row_id_base=0, ctx=""):
    in_rp = ref["in_rp"].astype(bool)
    rows = np.nonzero(in_rp)[0]
    assert np.array_equal(g["row"], rows + row_id_base), (ctx, "level-1 rows")
    lens_g = np.diff(g["offsets"])
    assert np.array_equal(lens_g, ref["lens"][rows]), (ctx, "level-1 lengths")
    assert g["offsets"][-1] == len(g["values"]) == len(ref["values"]), ctx
    # owner of every level-2 slot is the level-1 entry that holds it
    assert np.array_equal(g["owner"], np.repeat(g["row"], lens_g)), (ctx, "owner")
    for k, r in enumerate(rows):
        got = np.sort(g["values"][g["offsets"][k]:g["offsets"][k + 1]])
        exp = np.sort(ref["values"][ref["offsets"][r]:ref["offsets"][r + 1]])
        if not np.array_equal(got, exp):
            raise AssertionError("%s row %d: gpu %s oracle %s" % (ctx, r, got[:8], exp[:8]))


@pytest.mark.parametrize("seed", [1, 2])
def test_collect_nulls_predicates_all_ops(eng, seed):
    t = query1.random_small(seed, n_r=3001, n_s=2003, key_hi=700, val_lo=-50, val_hi=50, null_frac=0.1)
    for corr_op in PLAN_OPS:
        plan = make_plan(corr_op, "min", "=", outer_preds=[{"col": "col3", "op": "<=", "lit": 1}],
                         inner_preds=[{"col": "col3", "op": "!=", "rhs": "col2"}])
        assert_collect_parity(gpu_collect(eng, t, plan, row_id_base=1000), oracle.collect(t, plan), 1000,
                              ctx=(seed, corr_op))


def test_collect_widths_and_composite(eng):
    rng = np.random.Generator(np.random.PCG64(5))
    big = lambda n: rng.integers(-2**40, 2**40, n, dtype=np.int64)  # noqa: E731
    keys = big(60)
    t = {"R": {"col1": keys[rng.integers(0, 60, 2500)], "col2": big(2500)},
         "S": {"col1": keys[rng.integers(0, 60, 2600)], "col2": big(2600)},
         "S_valid": {"col2": (rng.random(2600) > 0.05).astype(np.uint8)}}
    dt = {"R": {"col1": "int64", "col2": "int64"}, "S": {"col1": "int64", "col2": "int64"}}
    for corr_op in ("=", "<", "!="):
        plan = make_plan(corr_op, "min", "=")
        assert_collect_parity(gpu_collect(eng, t, plan, dtypes=dt), oracle.collect(t, plan), ctx=("i64", corr_op))
    t2 = query1.random_small(6, n_r=4000, n_s=5000, key_hi=30, null_frac=0.0)
    plan = make_plan("=", "min", "=", outer_key=["col1", "col3"], inner_key=["col1", "col3"])
    assert_collect_parity(gpu_collect(eng, t2, plan), oracle.collect(t2, plan), ctx="composite")


def test_collect_c2_shaped(eng):
    """C2's distributions (keys U[0, n/4): ~4 S rows per key) at 60,013 rows;
    '=' lists of ~4 values; '>' lists averaging |S|/2 are checked on an
    oracle-independent closed form (lengths = prefix counts)."""
    n = 60013
    t = query1.tables(n_r=n, n_s=n, key_hi=n // 4, val_hi=16, seed=2)
    plan = make_plan("=", "min", "=")
    assert_collect_parity(gpu_collect(eng, t, plan), oracle.collect(t, plan), ctx="C2 =")
    small = query1.tables(n_r=3000, n_s=4000, key_hi=1000, val_hi=16, seed=3)
    plan = make_plan(">", "min", "=")
    g = gpu_collect(eng, small, plan)
    assert_collect_parity(g, oracle.collect(small, plan), ctx="C2-shaped >")
    lens = np.diff(g["offsets"])
    _, _, cnt, _ = ind.closed_form(small["R"]["col1"], small["S"]["col1"], small["S"]["col2"], ">", "count")
    assert np.array_equal(lens, cnt)


def test_collect_degenerate(eng):
    t = query1.random_small(9, n_r=500, n_s=400, null_frac=0.0)
    # everything filtered on the outer side; no S row qualifies
    for plan in (make_plan("=", "min", "=", outer_preds=[{"col": "col3", "op": ">", "lit": 99}]),
                 make_plan("=", "min", "=", inner_preds=[{"col": "col3", "op": ">", "lit": 99}])):
        assert_collect_parity(gpu_collect(eng, t, plan), oracle.collect(t, plan), ctx="degenerate")
    empty = {"R": {"col1": np.zeros(0, np.int32), "col2": np.zeros(0, np.int32)},
             "S": {"col1": np.zeros(0, np.int32), "col2": np.zeros(0, np.int32)}}
    plan = make_plan("<", "min", "=")
    g = gpu_collect(eng, empty, plan)
    assert len(g["row"]) == 0 and len(g["values"]) == 0


def test_collect_requires_index(eng):
    t = query1.random_small(3, n_r=10, n_s=10, null_frac=0.0)
    m = eng.mark()
    try:
        R, S = load(eng, t)
        with pytest.raises(NestGPUError) as e:
            eng.exec_collect(make_plan("=", "min", "="), R, S, -1)
        assert e.value.code == ERR_UNSUPPORTED
        idx = eng.build_index(S, ["col1"], payload=None)
        with pytest.raises(NestGPUError) as e:
            eng.exec_collect(make_plan("=", "min", "="), R, S, idx)
        assert e.value.code == ERR_INVALID
    finally:
        eng.release(m)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_collection_in(eng, seed):
    """R.col2 IN (SELECT S.col2 FROM S WHERE ... R.col1 OP S.col1): GPU vs the
    oracle's two-level arrays and SQLite's literal IN."""
    t = query1.random_small(seed + 40, n_r=2000, n_s=1500, key_hi=300, val_lo=-6, val_hi=6, null_frac=0.1)
    con = ind._db(t)
    for corr_op in PLAN_OPS:
        plan = make_plan(corr_op, "min", "=", inner_preds=[{"col": "col3", "op": ">=", "lit": 1}],
                         outer_preds=[{"col": "col3", "op": "!=", "lit": 2}])
        in_rp, passed = oracle.in_list(t, plan, "col2")
        m = eng.mark()
        try:
            R, S = load(eng, t)
            idx = eng.build_index(S, ["col1"], payload="col2", inner_preds=plan["inner_preds"])
            coll = eng.exec_collect(plan, R, S, idx)
            surv = eng.result_to_numpy(eng.collection_in(coll, R["col2"]))
            coll = eng.exec_collect(plan, R, S, idx)
            allr = eng.result_to_numpy(eng.collection_in(coll, R["col2"], emit_all=True))
        finally:
            eng.release(m)
        exp = np.nonzero(passed)[0]
        assert np.array_equal(surv["row"], exp), corr_op
        assert np.all(surv["value"] == 1) and np.all(surv["passed"] == 1)
        assert exp.tolist() == ind.in_sqlite(t, plan, "col2", con), corr_op
        assert np.array_equal(allr["row"], np.nonzero(in_rp)[0])
        assert np.array_equal(allr["passed"], passed[in_rp.astype(bool)])


def test_column_from_device(eng):
    torch = pytest.importorskip("torch")
    m = eng.mark()
    try:
        src = torch.tensor([5, -7, 2**31 - 1, -2**31, 0], dtype=torch.int64, device="cuda")
        vld = torch.tensor([1, 1, 1, 1, 0], dtype=torch.uint8, device="cuda")
        c = eng.column_from_device(src.data_ptr(), 5, "int32", d_valid=vld.data_ptr())
        info = eng.column_info(c)
        v = eng.arena_view(info["d_values"], 20).view(torch.int32).cpu().numpy()
        ok = eng.arena_view(info["d_valid"], 5).cpu().numpy()
        assert v.tolist() == [5, -7, 2**31 - 1, -2**31, 0] and ok.tolist() == [1, 1, 1, 1, 0]
        big = torch.tensor([1, 2**31], dtype=torch.int64, device="cuda")
        with pytest.raises(NestGPUError) as e:
            eng.column_from_device(big.data_ptr(), 2, "int32")
        assert e.value.code == ERR_OVERFLOW
        # an out-of-range value under a NULL mask is not an overflow
        nul = torch.tensor([1, 0], dtype=torch.uint8, device="cuda")
        eng.column_from_device(big.data_ptr(), 2, "int32", d_valid=nul.data_ptr())
        c64 = eng.column_from_device(big.data_ptr(), 2, "int64")
        assert eng.column_info(c64)["d_valid"] is None
        torch.cuda.synchronize()
    finally:
        eng.release(m)


# ------------------------------------------------------------------ Fig. 5 joins with subqueries
def _sqlite(tables):
    con = sqlite3.connect(":memory:")
    for name, cols in tables.items():
        names = [c for c in cols if c != "rid"]
        n = len(cols[names[0]])
        con.execute("CREATE TABLE %s (rid INTEGER, %s)" % (name, ", ".join(c + " INTEGER" for c in names)))
        con.executemany("INSERT INTO %s VALUES (%s)" % (name, ",".join("?" * (len(names) + 1))),
                        [(i,) + tuple(int(cols[c][i]) for c in names) for i in range(n)])
    return con


def _join_tables(seed, nl, nr, ns, key_hi):
    rng = np.random.Generator(np.random.PCG64(seed))
    i32 = lambda n, lo, hi: rng.integers(lo, hi, size=n).astype(np.int32)  # noqa: E731
    L = {"col1": i32(nl, 0, 8), "col2": i32(nl, 0, key_hi), "a": i32(nl, 0, 40), "rid": np.arange(nl, dtype=np.int32)}
    RT = {"col1": i32(nr, 0, key_hi), "a": i32(nr, 0, 40)}
    S = {"k1": i32(ns, 0, key_hi), "k2": i32(ns, 0, key_hi), "v": i32(ns, 0, 8)}
    return L, RT, S


@pytest.mark.parametrize("mode", ["index", "bnl"])
def test_join_subquery_right(eng, mode):
    """Fig. 5 case 1: LEFT.col1 = SUBQ(RIGHT.col1)."""
    L, RT, S = _join_tables(11, 3000, 2000, 2500, 600)
    con = _sqlite({"L": L, "RT": RT, "S": S})
    exp = sorted(con.execute(
        "SELECT L.rid, RT.rid FROM L, RT WHERE L.col1 = "
        "(SELECT MIN(S.v) FROM S WHERE S.k1 = RT.col1)").fetchall())
    m = eng.mark()
    try:
        Ld = eng.load_table(L)
        Rd = eng.load_table(RT)
        Sd = eng.load_table(S)
        plan = make_plan("=", "min", "=", outer_key=["col1"], inner_key=["k1"], agg_col="v", outer_cmp_col="col1")
        a, b = nested.join_subquery_right(eng, Ld, "col1", "rid", Rd, Sd, plan, mode=mode)
    finally:
        eng.release(m)
    assert sorted(zip(a.tolist(), b.tolist())) == exp
    assert len(exp) > 1000   # the join is not trivially empty


@pytest.mark.parametrize("mode", ["index", "bnl"])
def test_join_subquery_both(eng, mode):
    """Fig. 5 case 2: LEFT.col1 = SUBQ(LEFT.col2, RIGHT.col1), joined on a."""
    L, RT, S = _join_tables(12, 2000, 1500, 3000, 12)
    con = _sqlite({"L": L, "RT": RT, "S": S})
    exp = sorted(con.execute(
        "SELECT L.rid, RT.rid FROM L, RT WHERE L.a = RT.a AND L.col1 = "
        "(SELECT MIN(S.v) FROM S WHERE S.k1 = L.col2 AND S.k2 = RT.col1)").fetchall())
    m = eng.mark()
    try:
        Ld = eng.load_table(L)
        Rd = eng.load_table(RT)
        Sd = eng.load_table(S)
        plan = make_plan("=", "min", "=", outer_key=["l.col2", "r.col1"], inner_key=["k1", "k2"], agg_col="v",
                         outer_cmp_col="l.col1")
        a, b = nested.join_subquery_both(eng, Ld, Rd, Sd, ("a", "a"), "rid", plan, mode=mode)
    finally:
        eng.release(m)
    assert sorted(zip(a.tolist(), b.tolist())) == exp
    assert len(exp) > 100
