"""Pins for the TPC-H-shaped workloads (CPU, -m "not gpu").

SQLite runs the ORIGINAL nested TPC-H SQL (Q2, Q4, Q17, Q20's correlated
block) on the dbgen-like base tables at SF 0.01, with real strings for
p_type / p_brand / p_container / p_name / r_name and LIKE; the oracle runs
the flattened template plan (datagen/tpch.py).  Agreement pins the flattening
(join-first P:227, invariant hoisting P:319-329, LIKE -> flags R10, dates R11,
multipliers R7, composite keys R9) independently of both the oracle and the
CUDA path.  Post-processing outside the correlated subquery (ORDER BY/LIMIT,
GROUP BY, /7.0) is not part of the hot path and not compared.
"""
import sqlite3

import numpy as np
import pytest

import oracle
from datagen import tpch

SF = 0.01


@pytest.fixture(scope="module")
def base():
    return tpch.base_tables(SF, seed=11)


@pytest.fixture(scope="module")
def db(base):
    T = base
    con = sqlite3.connect(":memory:")

    def put(name, cols, extra=None):
        names = list(cols) + (list(extra) if extra else [])
        data = [np.asarray(cols[c]).tolist() for c in cols] + ([extra[c] for c in extra] if extra else [])
        con.execute("CREATE TABLE %s (%s)" % (name, ", ".join(names)))
        con.executemany("INSERT INTO %s VALUES (%s)" % (name, ",".join("?" * len(names))), zip(*data))

    put("region", T["region"], {"r_name": tpch.REGIONS})
    put("nation", T["nation"], {"n_name": [n for n, _ in tpch.NATIONS]})
    put("supplier", T["supplier"])
    p = T["part"]
    put("part", p, {
        "p_type_s": ["%s %s %s" % (tpch.TYPE_S1[t // 25], tpch.TYPE_S2[(t // 5) % 5], tpch.TYPE_S3[t % 5])
                     for t in p["p_type"].tolist()],
        "p_brand_s": ["Brand#%d%d" % (b // 5 + 1, b % 5 + 1) for b in p["p_brand"].tolist()],
        "p_container_s": ["%s %s" % (tpch.CONT_S1[c // 8], tpch.CONT_S2[c % 8]) for c in p["p_container"].tolist()],
        "p_name": ["%s misc words" % tpch.COLORS[w] for w in p["p_name1"].tolist()],
    })
    put("partsupp", T["partsupp"])
    put("orders", T["orders"])
    put("lineitem", T["lineitem"])
    for stmt in ("CREATE INDEX li_pk ON lineitem(l_partkey, l_suppkey)", "CREATE INDEX li_ok ON lineitem(l_orderkey)",
                 "CREATE INDEX ps_pk ON partsupp(ps_partkey)", "CREATE INDEX s_k ON supplier(s_suppkey)",
                 "CREATE INDEX p_k ON part(p_partkey)"):
        con.execute(stmt)
    return con


def _oracle_rows(tables, plan):
    res = oracle.evaluate(tables, plan)
    return np.nonzero(res["passed"])[0]


def test_q2(base, db):
    tables, plan = tpch.q2(base)
    rows = _oracle_rows(tables, plan)
    got = sorted(zip(base["partsupp"]["ps_partkey"][rows].tolist(), base["partsupp"]["ps_suppkey"][rows].tolist()))
    sql = """
      SELECT p_partkey, s_suppkey FROM part, supplier, partsupp, nation, region
      WHERE p_partkey = ps_partkey AND s_suppkey = ps_suppkey AND p_size = 15 AND p_type_s LIKE '%BRASS'
        AND s_nationkey = n_nationkey AND n_regionkey = r_regionkey AND r_name = 'EUROPE'
        AND ps_supplycost = (SELECT min(ps_supplycost) FROM partsupp, supplier, nation, region
                             WHERE p_partkey = ps_partkey AND s_suppkey = ps_suppkey
                               AND s_nationkey = n_nationkey AND n_regionkey = r_regionkey
                               AND r_name = 'EUROPE')"""
    exp = sorted(db.execute(sql).fetchall())
    assert got == exp and len(exp) > 0


@pytest.mark.parametrize("with_brand", [True, False])
def test_q5_non_unnestable(with_brand):
    """Query 5: Q2 (+ Brand#41) with ps_supplycost > MIN and the
    correlation p_partkey != ps_partkey.  SF 0.2 without lineitem/orders;
    the brand-less variant keeps ~100 outer rows."""
    T = tpch.base_tables(0.2, seed=12)
    con = sqlite3.connect(":memory:")
    for name, cols in (("supplier", T["supplier"]), ("partsupp", T["partsupp"])):
        con.execute("CREATE TABLE %s (%s)" % (name, ", ".join(cols)))
        con.executemany("INSERT INTO %s VALUES (%s)" % (name, ",".join("?" * len(cols))),
                        zip(*[c.tolist() for c in cols.values()]))
    con.execute("CREATE TABLE nation (n_nationkey, n_regionkey)")
    con.executemany("INSERT INTO nation VALUES (?,?)", zip(range(25), [r for _, r in tpch.NATIONS]))
    con.execute("CREATE TABLE region (r_regionkey, r_name)")
    con.executemany("INSERT INTO region VALUES (?,?)", enumerate(tpch.REGIONS))
    p = T["part"]
    con.execute("CREATE TABLE part (p_partkey, p_size, p_type_s, p_brand_s)")
    con.executemany("INSERT INTO part VALUES (?,?,?,?)", zip(
        p["p_partkey"].tolist(), p["p_size"].tolist(),
        ["%s %s %s" % (tpch.TYPE_S1[t // 25], tpch.TYPE_S2[(t // 5) % 5], tpch.TYPE_S3[t % 5]) for t in p["p_type"].tolist()],
        ["Brand#%d%d" % (b // 5 + 1, b % 5 + 1) for b in p["p_brand"].tolist()]))
    con.execute("CREATE INDEX s_k ON supplier(s_suppkey)")
    tables, plan = tpch.q5(T)
    if not with_brand:
        plan = dict(plan, outer_preds=[q for q in plan["outer_preds"] if q["col"] != "p_brand"])
    rows = _oracle_rows(tables, plan)
    got = sorted(zip(T["partsupp"]["ps_partkey"][rows].tolist(), T["partsupp"]["ps_suppkey"][rows].tolist()))
    sql = """
      SELECT p_partkey, s_suppkey FROM part, supplier, partsupp, nation, region
      WHERE p_partkey = ps_partkey AND s_suppkey = ps_suppkey AND p_size = 15 AND p_type_s LIKE '%%BRASS'
        %s
        AND s_nationkey = n_nationkey AND n_regionkey = r_regionkey AND r_name = 'EUROPE'
        AND ps_supplycost > (SELECT min(ps_supplycost) FROM partsupp, supplier, nation, region
                             WHERE p_partkey != ps_partkey AND s_suppkey = ps_suppkey
                               AND s_nationkey = n_nationkey AND n_regionkey = r_regionkey
                               AND r_name = 'EUROPE')""" % ("AND p_brand_s = 'Brand#41'" if with_brand else "")
    exp = sorted(con.execute(sql).fetchall())
    assert got == exp and len(exp) > 0


def test_q17(base, db):
    tables, plan = tpch.q17(base)
    rows = _oracle_rows(tables, plan)
    sql = """
      SELECT l.rowid - 1 FROM lineitem l, part
      WHERE p_partkey = l.l_partkey AND p_brand_s = 'Brand#23' AND p_container_s = 'MED BOX'
        AND 5 * l.l_quantity < (SELECT avg(l_quantity) FROM lineitem WHERE l_partkey = p_partkey)"""
    exp = sorted(r for (r,) in db.execute(sql))
    assert rows.tolist() == exp and len(exp) > 0


def test_q4(base, db):
    tables, plan = tpch.q4(base)
    rows = _oracle_rows(tables, plan)
    sql = """
      SELECT o.rowid - 1 FROM orders o
      WHERE o_orderdate >= %d AND o_orderdate < %d
        AND EXISTS (SELECT * FROM lineitem WHERE l_orderkey = o_orderkey AND l_commitdate < l_receiptdate)""" % (
        tpch.D_1993_07_01, tpch.D_1993_10_01)
    exp = sorted(r for (r,) in db.execute(sql))
    assert rows.tolist() == exp and len(exp) > 0


def test_q20(base, db):
    tables, plan = tpch.q20(base)
    rows = _oracle_rows(tables, plan)
    sql = """
      SELECT ps.rowid - 1 FROM partsupp ps
      WHERE ps_partkey IN (SELECT p_partkey FROM part WHERE p_name LIKE 'forest%%')
        AND 200 * ps_availqty > (SELECT sum(l_quantity) FROM lineitem
                                 WHERE l_partkey = ps_partkey AND l_suppkey = ps_suppkey
                                   AND l_shipdate >= %d AND l_shipdate < %d)""" % (
        tpch.D_1994_01_01, tpch.D_1995_01_01)
    exp = sorted(r for (r,) in db.execute(sql))
    assert rows.tolist() == exp and len(exp) > 0


def test_base_table_shapes(base):
    T = base
    assert len(T["partsupp"]["ps_partkey"]) == 4 * len(T["part"]["p_partkey"])
    # 4 distinct suppliers per part (spec formula)
    pairs = set(zip(T["partsupp"]["ps_partkey"].tolist(), T["partsupp"]["ps_suppkey"].tolist()))
    assert len(pairs) == len(T["partsupp"]["ps_partkey"])
    li = T["lineitem"]
    assert np.all(li["l_receiptdate"] > li["l_shipdate"])
    assert set(zip(li["l_partkey"].tolist(), li["l_suppkey"].tolist())) <= pairs
    assert 1 <= len(li["l_orderkey"]) / len(T["orders"]["o_orderkey"]) <= 7


def test_q20_three_levels(base, db):
    """Full TPC-H Q20 (three nesting levels, Fig. 6) by the oracle,
    level by level (level-1 survivors' ps_suppkey feed level 0's IN), against
    SQLite running the original nested SQL."""
    tables1, plan1, carry, R0, plan0 = tpch.q20_levels(base)
    r1 = oracle.evaluate(tables1, plan1)
    rows1 = np.nonzero(r1["passed"])[0]
    S0 = {"ps_suppkey": tables1["R"][carry][rows1]}
    r0 = oracle.evaluate({"R": R0, "S": S0}, plan0)
    got = sorted(R0["s_suppkey"][np.nonzero(r0["passed"])[0]].tolist())
    sql = """
      SELECT s_suppkey FROM supplier, nation
      WHERE s_suppkey IN (
              SELECT ps_suppkey FROM partsupp
              WHERE ps_partkey IN (SELECT p_partkey FROM part WHERE p_name LIKE 'forest%%')
                AND 200 * ps_availqty > (SELECT sum(l_quantity) FROM lineitem
                                         WHERE l_partkey = ps_partkey AND l_suppkey = ps_suppkey
                                           AND l_shipdate >= %d AND l_shipdate < %d))
        AND s_nationkey = n_nationkey AND n_name = 'CANADA'""" % (tpch.D_1994_01_01, tpch.D_1995_01_01)
    exp = sorted(r for (r,) in db.execute(sql))
    assert got == exp and len(exp) > 0
