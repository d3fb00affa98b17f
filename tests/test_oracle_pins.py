"""Pins for the CPU oracle (oracle/), all CPU-only (-m "not gpu").

Each test checks the oracle against something other than itself:
  * a hand-worked Query 1 instance (tests/golden/query1_worked.json),
  * SQLite running the literal nested SQL, exhaustively over every single-row
    R against every S of <= 3 rows drawn from {0,1,2,NULL}^2 (reading R1/R2),
  * Query 2 (Kim's GROUP BY + JOIN unnesting) for '=',
  * the COUNT bug (reading R3) as a regression Query 2 must fail,
  * closed-form prefix / group aggregates for every operator,
  * invariants between operators and aggregates,
  * the pure-Python twin (exact Python ints / Fractions).
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle
from datagen import make_plan, PLAN_OPS, query1
from oracle import twin
from tests import independent as ind

GOLD = os.path.join(os.path.dirname(__file__), "golden", "query1_worked.json")
VALUE_AGGS = ("min", "max", "sum", "count", "avg")


def test_golden_worked_example(oracle_lib):
    g = json.load(open(GOLD))
    tables = {"R": {k: np.array(v, np.int32) for k, v in g["R"].items()},
              "S": {k: np.array(v, np.int32) for k, v in g["S"].items()}}
    for c in g["cases"]:
        plan = make_plan(c["corr_op"], c["agg"], c["outer_op"])
        res = oracle.evaluate(tables, plan)
        got = [int(v) if ok else None for v, ok in zip(res["value"], res["valid"])]
        assert got == c["subq"], c
        assert list(np.nonzero(res["passed"])[0]) == c["survivors"], c


# ---------------------------------------------------------------- SQLite exhaustive
_DOM = [0, 1, 2, None]


def _instances():
    pairs = list(itertools.product(_DOM, _DOM))
    s_tables = [()]
    for k in (1, 2, 3):
        s_tables += list(itertools.product(pairs, repeat=k))
    r_rows = pairs
    R = {"key": [], "cmp": []}
    S = {"key": [], "val": []}
    lo, hi = [], []
    for rk, rc in r_rows:
        for st in s_tables:
            R["key"].append(rk)
            R["cmp"].append(rc)
            lo.append(len(S["key"]))
            for sk, sv in st:
                S["key"].append(sk)
                S["val"].append(sv)
            hi.append(len(S["key"]))

    def enc(d):
        return ({c: np.array([0 if x is None else x for x in v], np.int64) for c, v in d.items()},
                {c: np.array([x is not None for x in v], np.uint8) for c, v in d.items()})

    Rv, Rm = enc(R)
    Sv, Sm = enc(S)
    gid_r = np.arange(len(lo), dtype=np.int64)
    gid_s = np.repeat(gid_r, np.array(hi) - np.array(lo))
    return {"R": Rv, "R_valid": Rm, "S": Sv, "S_valid": Sm}, gid_r, gid_s, np.array(lo), np.array(hi)


@pytest.fixture(scope="module")
def exhaustive():
    import sqlite3
    t, gid_r, gid_s, lo, hi = _instances()
    con = sqlite3.connect(":memory:")
    con.execute("CREATE TABLE R (rid INTEGER PRIMARY KEY, key INTEGER, cmp INTEGER)")
    con.execute("CREATE TABLE S (gid INTEGER, key INTEGER, val INTEGER)")
    nn = lambda v, m: [None if not mm else int(x) for x, mm in zip(v, m)]  # noqa: E731
    con.executemany("INSERT INTO R VALUES (?,?,?)",
                    zip(gid_r.tolist(), nn(t["R"]["key"], t["R_valid"]["key"]),
                        nn(t["R"]["cmp"], t["R_valid"]["cmp"])))
    con.executemany("INSERT INTO S VALUES (?,?,?)",
                    zip(gid_s.tolist(), nn(t["S"]["key"], t["S_valid"]["key"]),
                        nn(t["S"]["val"], t["S_valid"]["val"])))
    con.execute("CREATE INDEX s_gid ON S(gid)")
    return t, con, lo, hi


def _sql_nested(con, corr_op, agg, outer_op, a, b):
    op = ind.SQL_OP
    w = "S.gid = R.rid AND R.key %s S.key" % op[corr_op]
    sub = lambda e: "(SELECT %s FROM S WHERE %s)" % (e, w)  # noqa: E731
    if agg in ("exists", "not_exists"):
        cond = ("EXISTS " if agg == "exists" else "NOT EXISTS ") + sub("1")
    elif agg == "avg":
        cond = "%d*R.cmp*%s %s %d*%s" % (a, sub("COUNT(S.val)"), op[outer_op], b, sub("SUM(S.val)"))
    else:
        e = "COUNT(*)" if agg == "count" else "%s(S.val)" % agg.upper()
        cond = "%d*R.cmp %s %d*%s" % (a, op[outer_op], b, sub(e))
    return set(r for (r,) in con.execute("SELECT rid FROM R WHERE " + cond))


def _sql_values(con, corr_op, agg):
    w = "S.gid = R.rid AND R.key %s S.key" % ind.SQL_OP[corr_op]
    if agg == "avg":
        rows = con.execute("SELECT rid, (SELECT SUM(val) FROM S WHERE %s), "
                           "(SELECT COUNT(val) FROM S WHERE %s) FROM R ORDER BY rid" % (w, w)).fetchall()
        return [(s, c) for _, s, c in rows]
    if agg in ("exists", "not_exists"):
        e = "CASE WHEN %sEXISTS (SELECT 1 FROM S WHERE %s) THEN 1 ELSE 0 END" % (
            "" if agg == "exists" else "NOT ", w)
    else:
        e = "(SELECT %s FROM S WHERE %s)" % ("COUNT(*)" if agg == "count" else "%s(val)" % agg.upper(), w)
    return [v for _, v in con.execute("SELECT rid, %s FROM R ORDER BY rid" % e)]


@pytest.mark.parametrize("corr_op", PLAN_OPS)
def test_sqlite_exhaustive(exhaustive, oracle_lib, corr_op):
    t, con, lo, hi = exhaustive
    for agg in VALUE_AGGS + ("exists", "not_exists"):
        plan0 = make_plan(corr_op, agg, "=", outer_key=["key"], inner_key=["key"],
                          agg_col="val", outer_cmp_col="cmp")
        # subquery values
        res = oracle.evaluate(t, plan0, s_window=(lo, hi))
        sv = _sql_values(con, corr_op, agg)
        if agg == "avg":
            for i, (s, c) in enumerate(sv):
                if c:
                    assert res["valid"][i] and res["sum"][i] == s and res["cnt"][i] == c
                    assert res["value"][i] == ind.round_half_away(ind.Fraction(s * 10 ** 6, c))
                else:
                    assert not res["valid"][i]
        else:
            exp_valid = np.array([v is not None for v in sv])
            exp_val = np.array([0 if v is None else v for v in sv], np.int64)
            assert np.array_equal(res["valid"].astype(bool), exp_valid), (corr_op, agg)
            assert np.array_equal(res["value"], exp_val), (corr_op, agg)
        # survivors for each outer operator and two multiplier settings
        outer_ops = ("=",) if agg in ("exists", "not_exists") else PLAN_OPS
        for outer_op in outer_ops:
            for a, b in ((1, 1), (3, 2)):
                plan = dict(plan0, outer_op=outer_op, lhs_mult=a, rhs_mult=b)
                res = oracle.evaluate(t, plan, s_window=(lo, hi))
                got = set(np.nonzero(res["passed"])[0].tolist())
                exp = _sql_nested(con, corr_op, agg, outer_op, a, b)
                assert got == exp, (corr_op, agg, outer_op, a, b, sorted(got ^ exp)[:5])


# ---------------------------------------------------------------- local predicates
@pytest.mark.parametrize("seed", range(6))
def test_sqlite_random_with_predicates(oracle_lib, seed):
    rng = np.random.default_rng(seed)
    t = query1.random_small(seed, n_r=40, n_s=30)
    con = ind._db(t)
    for corr_op in PLAN_OPS:
        for agg in VALUE_AGGS + ("exists", "not_exists"):
            op = PLAN_OPS[rng.integers(6)]
            plan = make_plan(corr_op, agg, op,
                             outer_preds=[{"col": "col3", "op": "<=", "lit": 1}],
                             inner_preds=[{"col": "col3", "op": "!=", "rhs": "col2"}],
                             lhs_mult=int(rng.integers(1, 4)), rhs_mult=int(rng.integers(1, 4)))
            res = oracle.evaluate(t, plan)
            surv, vals, avg = ind.nested_sqlite(t, plan, con)
            assert sorted(np.nonzero(res["passed"])[0].tolist()) == surv, (corr_op, agg)
            for rid, v in vals.items():
                assert res["in_rp"][rid]
                if v is None:
                    assert not res["valid"][rid]
                else:
                    assert res["valid"][rid] and res["value"][rid] == v, (corr_op, agg, rid)
            inrp = set(np.nonzero(res["in_rp"])[0].tolist())
            assert inrp == set(vals) | set(avg) or agg == "avg" and inrp == set(avg)


def test_composite_key_against_sqlite(oracle_lib):
    t = query1.random_small(11, n_r=50, n_s=60, key_hi=3)
    con = ind._db(t)
    for agg in VALUE_AGGS + ("exists",):
        plan = make_plan("=", agg, "<=", outer_key=["col1", "col3"], inner_key=["col1", "col3"])
        res = oracle.evaluate(t, plan)
        surv, vals, _ = ind.nested_sqlite(t, plan, con)
        assert sorted(np.nonzero(res["passed"])[0].tolist()) == surv, agg


# ---------------------------------------------------------------- Query 1 == Query 2
@pytest.mark.parametrize("agg", ["min", "max", "sum"])
def test_query2_equivalence(oracle_lib, agg):
    """P:37 / P:109: Kim's unnesting (Query 2) returns the same multiset as
    the nested Query 1 for '=' with MIN (and MAX/SUM likewise)."""
    t = query1.tables(n_r=20000, n_s=20000, key_hi=5000, val_hi=16, seed=3,
                      empty_frac=0.1, empty_hi=5500)
    if agg == "sum":
        t["R"]["col2"] = t["R"]["col2"] * 3  # sums of ~4 values in [0,16)
    plan = make_plan("=", agg, "=")
    res = oracle.evaluate(t, plan)
    rows, _ = oracle.survivors(res)
    nested = sorted(zip(t["R"]["col1"][rows].tolist(), t["R"]["col2"][rows].tolist()))
    assert nested == ind.query2_sqlite(t, agg)
    assert len(nested) > 100


def test_count_bug(oracle_lib):
    """Reading R3: for COUNT the nested form keeps r with no match and
    R.col2 = 0; Query 2's join drops it (Kim's COUNT bug)."""
    t = {"R": {"col1": np.array([1, 7], np.int32), "col2": np.array([1, 0], np.int32)},
         "S": {"col1": np.array([1, 2], np.int32), "col2": np.array([5, 6], np.int32)}}
    res = oracle.evaluate(t, make_plan("=", "count", "="))
    assert res["passed"].tolist() == [1, 1]
    q2 = ind._db(t).execute("SELECT R.rid FROM R, (SELECT COUNT(*) AS c, col1 FROM S GROUP BY col1) T "
                            "WHERE R.col1 = T.col1 AND R.col2 = T.c").fetchall()
    assert q2 == [(0,)]  # Query 2 loses row 1


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("corr_op", PLAN_OPS)
def test_closed_form(oracle_lib, corr_op):
    t = query1.tables(n_r=3001, n_s=20011, key_hi=4000, val_hi=1000, seed=5)
    t["S"]["col2"] = t["S"]["col2"] - 500   # negative values too
    for agg in VALUE_AGGS + ("exists", "not_exists"):
        res = oracle.evaluate(t, make_plan(corr_op, agg, "<"))
        valid, value, cnt, ssum = ind.closed_form(t["R"]["col1"], t["S"]["col1"], t["S"]["col2"],
                                                  corr_op, agg)
        assert np.array_equal(res["valid"].astype(bool), valid), (corr_op, agg)
        assert np.array_equal(res["value"], value), (corr_op, agg)
        if agg == "avg":
            assert np.array_equal(res["cnt"][valid], cnt[valid])
            assert np.array_equal(res["sum"][valid], ssum[valid])
        if agg not in ("exists", "not_exists"):
            x = t["R"]["col2"].astype(np.int64)
            if agg == "avg":
                exp = valid & (x * cnt < ssum)
            else:
                exp = valid & (x < value)
            assert np.array_equal(res["passed"].astype(bool), exp), (corr_op, agg)


def test_invariants(oracle_lib):
    t = query1.tables(n_r=2000, n_s=5000, key_hi=700, val_hi=50, seed=9)
    c = {op: oracle.evaluate(t, make_plan(op, "count", "="))["value"] for op in PLAN_OPS}
    n = len(t["S"]["col1"])
    assert np.array_equal(c["<"] + c["="] + c[">"], np.full(2000, n))
    assert np.array_equal(c["!="], n - c["="])
    assert np.array_equal(c["<="], c["<"] + c["="])
    assert np.array_equal(c[">="], c[">"] + c["="])
    for op in PLAN_OPS:
        ex = oracle.evaluate(t, make_plan(op, "exists", "="))["value"]
        nex = oracle.evaluate(t, make_plan(op, "not_exists", "="))["value"]
        assert np.array_equal(ex, (c[op] > 0).astype(np.int64))
        assert np.array_equal(nex, 1 - ex)
        mn = oracle.evaluate(t, make_plan(op, "min", "="))
        mx = oracle.evaluate(t, make_plan(op, "max", "="))
        av = oracle.evaluate(t, make_plan(op, "avg", "="))
        sm = oracle.evaluate(t, make_plan(op, "sum", "="))
        ok = av["valid"].astype(bool)
        assert np.array_equal(ok, c[op] > 0)
        assert np.all(mn["value"][ok] * 10 ** 6 <= av["value"][ok])
        assert np.all(av["value"][ok] <= mx["value"][ok] * 10 ** 6)
        assert np.array_equal(av["sum"][ok], sm["value"][ok])
        assert np.array_equal(av["cnt"][ok], c[op][ok])


def test_sampled_rows_match_full(oracle_lib):
    t = query1.tables(n_r=3000, n_s=3000, key_hi=900, val_hi=16, seed=4)
    plan = make_plan(">", "min", "=")
    full = oracle.evaluate(t, plan)
    rows = np.array([0, 17, 2999, 1500, 17], np.int64)
    part = oracle.evaluate(t, plan, rows=rows)
    for k in ("passed", "valid", "value"):
        assert np.array_equal(part[k], full[k][rows])


def test_twin_agrees(oracle_lib):
    """C oracle == pure-Python twin (exact ints / Fractions) on random tiny
    tables with NULLs, negative values and local predicates."""
    for seed in range(4):
        t = query1.random_small(100 + seed, n_r=25, n_s=20)
        for corr_op in PLAN_OPS:
            for agg in VALUE_AGGS + ("exists", "not_exists"):
                plan = make_plan(corr_op, agg, PLAN_OPS[seed % 6],
                                 outer_preds=[{"col": "col3", "op": "!=", "lit": 2}],
                                 inner_preds=[{"col": "col2", "op": ">=", "rhs": "col3"}],
                                 lhs_mult=2, rhs_mult=1 + seed)
                res = oracle.evaluate(t, plan)
                tw = twin.evaluate(t, plan)
                for k in ("in_rp", "passed", "valid", "value", "sum", "cnt"):
                    assert res[k].tolist() == [d[k] for d in tw], (corr_op, agg, k)


def test_overflow_detected(oracle_lib):
    big = np.array([2 ** 62, 2 ** 62, 2 ** 62], np.int64)
    t = {"R": {"k": np.array([0], np.int64), "x": np.array([0], np.int64)},
         "S": {"k": np.zeros(3, np.int64), "v": big}}
    with pytest.raises(oracle.OracleOverflow):
        oracle.evaluate(t, make_plan("=", "sum", "=", outer_key=["k"], inner_key=["k"],
                                     agg_col="v", outer_cmp_col="x"))


# ---------------------------------------------------------------- type-J two-level arrays
@pytest.mark.parametrize("seed", range(4))
def test_collect_against_sqlite_join(oracle_lib, seed):
    """oracle.collect (P:231 two-level arrays) vs SQLite running the unnested
    JOIN form; NULL keys / payloads / local predicates included."""
    t = query1.random_small(100 + seed, n_r=40, n_s=35)
    con = ind._db(t)
    for corr_op in PLAN_OPS:
        plan = make_plan(corr_op, "min", "=",
                         outer_preds=[{"col": "col3", "op": "<=", "lit": 1}],
                         inner_preds=[{"col": "col3", "op": "!=", "lit": 0}])
        c = oracle.collect(t, plan)
        exp = ind.collect_sqlite(t, plan, con)
        assert set(np.nonzero(c["in_rp"])[0].tolist()) == set(exp)
        for r in range(len(c["lens"])):
            got = sorted(c["values"][c["offsets"][r]:c["offsets"][r + 1]].tolist())
            assert got == exp.get(r, []), (corr_op, r)


def test_collect_consistent_with_aggregates(oracle_lib):
    """Level 1 lengths == AVG's nn, and min / max / sum of each level-2 list ==
    the (pinned) MIN / MAX / SUM evaluations of the same subquery."""
    t = query1.random_small(7, n_r=60, n_s=80)
    for corr_op in PLAN_OPS:
        c = oracle.collect(t, make_plan(corr_op, "min", "="))
        ev = {a: oracle.evaluate(t, make_plan(corr_op, a, "=")) for a in ("min", "max", "sum", "avg")}
        assert np.array_equal(c["lens"], ev["avg"]["cnt"])
        for r in range(len(c["lens"])):
            lst = c["values"][c["offsets"][r]:c["offsets"][r + 1]]
            if len(lst):
                assert ev["min"]["value"][r] == lst.min() and ev["max"]["value"][r] == lst.max()
                assert ev["sum"]["value"][r] == lst.sum()
            else:
                assert not ev["min"]["valid"][r] and not ev["sum"]["valid"][r]


@pytest.mark.parametrize("seed", range(3))
def test_in_list_against_sqlite(oracle_lib, seed):
    """x IN (correlated type-J subquery) read off the two-level arrays vs
    SQLite's literal IN (NULL x, NULL elements, empty lists)."""
    t = query1.random_small(200 + seed, n_r=50, n_s=40)
    con = ind._db(t)
    for corr_op in PLAN_OPS:
        plan = make_plan(corr_op, "min", "=", inner_preds=[{"col": "col3", "op": ">=", "lit": 1}])
        in_rp, passed = oracle.in_list(t, plan, "col2")
        assert np.nonzero(passed)[0].tolist() == ind.in_sqlite(t, plan, "col2", con), corr_op


@pytest.mark.parametrize("outer_op", ["=", "!=", "<", "<=", ">", ">="])
def test_closed_form_outer_passed(oracle_lib, outer_op):
    """oracle/unnested.outer_passed (the full-size GPU tests' check of the
    outer comparison on every row) against the oracle's `passed`, with
    multipliers (reading R7) and every aggregate."""
    t = query1.tables(n_r=2003, n_s=5003, key_hi=600, val_hi=30, seed=11)
    for corr_op in ("=", "!=", ">"):
        for agg in VALUE_AGGS + ("count", "exists", "not_exists"):
            plan = make_plan(corr_op, agg, outer_op, lhs_mult=3, rhs_mult=2)
            res = oracle.evaluate(t, plan)
            valid, value, cnt, ssum = ind.closed_form(t["R"]["col1"], t["S"]["col1"], t["S"]["col2"], corr_op, agg)
            got = ind.outer_passed(t["R"]["col2"], valid, value, cnt, ssum, agg, outer_op, 3, 2)
            assert np.array_equal(res["passed"].astype(bool), got), (corr_op, agg, outer_op)
