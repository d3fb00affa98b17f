"""TPC-H-shaped base tables and their flattening into the plan template.

PAPER.md P:439-553 (§V-A) evaluates TPC-H Q2, Q4 and Q17 (type-JA / EXISTS
subqueries) on dbgen data; BASELINE.json configs[2..3] add Q20.  No dbgen or
network is available, so this module draws dbgen-LIKE columns from the TPC-H
specification's distributions (recalled, SURVEY.md §0 [TPC-H]; not
dbgen-exact, so official answers do not apply).  Strings are dictionary codes;
LIKE predicates become flag columns computed on the host (R10);
dates are int32 days since 1970-01-01 (R11); decimals are scaled integers.

Flattening = the paper's "join first, then selection with subquery"
and invariant hoisting, applied once on the host: every FK lookup
(partsupp->supplier->nation->region, lineitem->part, ...) is a numpy gather.
The result is the template's R (outer block) and S (inner block) plus a plan.

This module produces INPUTS only; no subquery arithmetic lives here.
"""
import datetime

import numpy as np

EPOCH = datetime.date(1970, 1, 1)


def day(y, m, d):
    return (datetime.date(y, m, d) - EPOCH).days


D_1992_01_01 = day(1992, 1, 1)      # 8035
D_1998_08_02 = day(1998, 8, 2)
D_1993_07_01 = day(1993, 7, 1)      # 8582  (Q4)
D_1993_10_01 = day(1993, 10, 1)     # 8674
D_1994_01_01 = day(1994, 1, 1)      # 8766  (Q20)
D_1995_01_01 = day(1995, 1, 1)      # 9131

REGIONS = ["AFRICA", "AMERICA", "ASIA", "EUROPE", "MIDDLE EAST"]
NATIONS = [("ALGERIA", 0), ("ARGENTINA", 1), ("BRAZIL", 1), ("CANADA", 1), ("EGYPT", 4), ("ETHIOPIA", 0),
           ("FRANCE", 3), ("GERMANY", 3), ("INDIA", 2), ("INDONESIA", 2), ("IRAN", 4), ("IRAQ", 4),
           ("JAPAN", 2), ("JORDAN", 4), ("KENYA", 0), ("MOROCCO", 0), ("MOZAMBIQUE", 0), ("PERU", 1),
           ("CHINA", 2), ("ROMANIA", 3), ("SAUDI ARABIA", 4), ("VIETNAM", 2), ("RUSSIA", 3),
           ("UNITED KINGDOM", 3), ("UNITED STATES", 1)]
TYPE_S1 = ["STANDARD", "SMALL", "MEDIUM", "LARGE", "ECONOMY", "PROMO"]
TYPE_S2 = ["ANODIZED", "BURNISHED", "PLATED", "POLISHED", "BRUSHED"]
TYPE_S3 = ["TIN", "NICKEL", "BRASS", "STEEL", "COPPER"]
CONT_S1 = ["SM", "LG", "MED", "JUMBO", "WRAP"]
CONT_S2 = ["CASE", "BOX", "BAG", "JAR", "PKG", "PACK", "CAN", "DRUM"]
PRIORITIES = ["1-URGENT", "2-HIGH", "3-MEDIUM", "4-NOT SPECIFIED", "5-LOW"]
COLORS = ["almond", "antique", "aquamarine", "azure", "beige", "bisque", "black", "blanched", "blue", "blush",
          "brown", "burlywood", "burnished", "chartreuse", "chiffon", "chocolate", "coral", "cornflower",
          "cornsilk", "cream", "cyan", "dark", "deep", "dim", "dodger", "drab", "firebrick", "floral", "forest",
          "frosted", "gainsboro", "ghost", "goldenrod", "green", "grey", "honeydew", "hot", "indian", "ivory",
          "khaki", "lace", "lavender", "lawn", "lemon", "light", "lime", "linen", "magenta", "maroon", "medium",
          "metallic", "midnight", "mint", "misty", "moccasin", "navajo", "navy", "olive", "orange", "orchid",
          "pale", "papaya", "peach", "peru", "pink", "plum", "powder", "puff", "purple", "red", "rose", "rosy",
          "royal", "saddle", "salmon", "sandy", "seashell", "sienna", "sky", "slate", "smoke", "snow", "spring",
          "steel", "tan", "thistle", "tomato", "turquoise", "violet", "wheat", "white", "yellow"]
assert len(COLORS) == 92

# dictionary codes used by the flattened plans
BRASS = TYPE_S3.index("BRASS")
EUROPE = REGIONS.index("EUROPE")
FOREST = COLORS.index("forest")


def brand_code(m, n):          # Brand#MN, M,N in 1..5
    return (m - 1) * 5 + (n - 1)


def container_code(s1, s2):
    return CONT_S1.index(s1) * len(CONT_S2) + CONT_S2.index(s2)


def base_tables(sf, seed):
    """dbgen-like base tables (int columns; decimals scaled by 100)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    i32 = np.int32
    n_supp = max(1, int(round(10000 * sf)))
    n_part = max(1, int(round(200000 * sf)))
    n_ord = max(1, int(round(1500000 * sf)))
    T = {}
    T["region"] = {"r_regionkey": np.arange(5, dtype=i32)}
    T["nation"] = {"n_nationkey": np.arange(25, dtype=i32),
                   "n_regionkey": np.array([r for _, r in NATIONS], dtype=i32)}
    T["supplier"] = {"s_suppkey": np.arange(1, n_supp + 1, dtype=i32),
                     "s_nationkey": rng.integers(0, 25, n_supp).astype(i32),
                     "s_acctbal": rng.integers(-99999, 999999, n_supp).astype(np.int64)}
    pk = np.arange(1, n_part + 1, dtype=np.int64)
    T["part"] = {
        "p_partkey": pk.astype(i32),
        "p_size": rng.integers(1, 51, n_part).astype(i32),
        "p_type": rng.integers(0, 150, n_part).astype(i32),         # s1*25 + s2*5 + s3
        "p_brand": rng.integers(0, 25, n_part).astype(i32),         # (M-1)*5 + (N-1)
        "p_container": rng.integers(0, 40, n_part).astype(i32),
        "p_name1": rng.integers(0, 92, n_part).astype(i32),         # first word of p_name
        # retail price (cents): (90000 + ((pk/10) % 20001) + 100*(pk % 1000))
        "p_retailprice": (90000 + (pk // 10) % 20001 + 100 * (pk % 1000)).astype(np.int64),
    }
    # partsupp: 4 suppliers per part, spec formula
    ps_pk = np.repeat(pk, 4)
    i = np.tile(np.arange(4, dtype=np.int64), n_part)
    S = n_supp
    ps_sk = (ps_pk + i * (S // 4 + (ps_pk - 1) // S)) % S + 1
    T["partsupp"] = {"ps_partkey": ps_pk.astype(i32), "ps_suppkey": ps_sk.astype(i32),
                     "ps_availqty": rng.integers(1, 10000, len(ps_pk)).astype(i32),
                     "ps_supplycost": rng.integers(100, 100001, len(ps_pk)).astype(i32)}   # cents
    # orders: sparse keys (8 of every 32), dates, priorities
    oi = np.arange(n_ord, dtype=np.int64)
    okey = (oi // 8) * 32 + (oi % 8) + 1
    odate = rng.integers(D_1992_01_01, D_1998_08_02 + 1, n_ord).astype(i32)
    T["orders"] = {"o_orderkey": okey.astype(np.int64), "o_orderdate": odate,
                   "o_orderpriority": rng.integers(0, 5, n_ord).astype(i32)}
    # lineitem: 1..7 lines per order
    nl = rng.integers(1, 8, n_ord)
    l_ord = np.repeat(np.arange(n_ord), nl)
    n_li = len(l_ord)
    l_pk = rng.integers(1, n_part + 1, n_li).astype(np.int64)
    li = rng.integers(0, 4, n_li)
    l_sk = (l_pk + li * (S // 4 + (l_pk - 1) // S)) % S + 1
    qty = rng.integers(1, 51, n_li).astype(np.int64)
    od = odate[l_ord].astype(np.int64)
    ship = od + rng.integers(1, 122, n_li)
    T["lineitem"] = {
        "l_orderkey": okey[l_ord].astype(np.int64),
        "l_partkey": l_pk.astype(i32),
        "l_suppkey": l_sk.astype(i32),
        "l_quantity": (qty * 100).astype(i32),                          # decimal(2) -> cents
        "l_extendedprice": (qty * T["part"]["p_retailprice"][l_pk - 1]).astype(np.int64),
        "l_shipdate": ship.astype(i32),
        "l_commitdate": (od + rng.integers(30, 91, n_li)).astype(i32),
        "l_receiptdate": (ship + rng.integers(1, 31, n_li)).astype(i32),
    }
    return T


# ------------------------------------------------------------------ flattening
def _plan(**kw):
    from .plans import make_plan
    return make_plan(**kw)


def q2(T):
    """TPC-H Q2: outer = part x partsupp x supplier x nation x region
    with p_size = 15, p_type LIKE '%BRASS', r_name = 'EUROPE'; inner =
    partsupp x supplier x nation x region with r_name = 'EUROPE';
    ps_supplycost = MIN(ps_supplycost) correlated on p_partkey = ps_partkey."""
    ps = T["partsupp"]
    part = T["part"]
    s_nat = T["supplier"]["s_nationkey"][ps["ps_suppkey"] - 1]
    s_reg = T["nation"]["n_regionkey"][s_nat]
    p_idx = ps["ps_partkey"] - 1
    R = {"p_partkey": ps["ps_partkey"], "ps_supplycost": ps["ps_supplycost"],
         "p_size": part["p_size"][p_idx], "p_brass": (part["p_type"][p_idx] % 5 == BRASS).astype(np.int32),
         "s_regionkey": s_reg.astype(np.int32)}
    S = {"ps_partkey": ps["ps_partkey"], "ps_supplycost": ps["ps_supplycost"], "s_regionkey": s_reg.astype(np.int32)}
    plan = _plan(corr_op="=", agg="min", outer_op="=", outer_key=["p_partkey"], inner_key=["ps_partkey"],
                 agg_col="ps_supplycost", outer_cmp_col="ps_supplycost",
                 outer_preds=[{"col": "p_size", "op": "=", "lit": 15}, {"col": "p_brass", "op": "=", "lit": 1},
                              {"col": "s_regionkey", "op": "=", "lit": EUROPE}],
                 inner_preds=[{"col": "s_regionkey", "op": "=", "lit": EUROPE}])
    return {"R": R, "S": S}, plan


def q5(T):
    """The paper's Query 5 (Fig. 11): TPC-H Q2 (+ Query 4's
    p_brand = 'Brand#41') with the subquery predicate changed to
    ps_supplycost > (...) and the correlation to p_partkey != ps_partkey --
    "cannot be unnested".  The diff in the paper is garbled
    (R13); this reading keeps Q2's other predicates."""
    tables, plan = q2(T)
    part = T["part"]
    tables["R"]["p_brand"] = part["p_brand"][T["partsupp"]["ps_partkey"] - 1]
    plan = dict(plan, corr_op="!=", outer_op=">",
                outer_preds=plan["outer_preds"] + [{"col": "p_brand", "op": "=", "lit": brand_code(4, 1)}])
    return tables, plan


def q17(T):
    """TPC-H Q17: outer = lineitem x part with p_brand = 'Brand#23'
    and p_container = 'MED BOX'; l_quantity < 0.2 * AVG(l_quantity) over the
    lineitems of the same part -> 5*l_quantity < avg (lhs_mult = 5, R7)."""
    li = T["lineitem"]
    part = T["part"]
    p_idx = li["l_partkey"] - 1
    R = {"l_partkey": li["l_partkey"], "l_quantity": li["l_quantity"],
         "p_brand": part["p_brand"][p_idx], "p_container": part["p_container"][p_idx]}
    S = {"l_partkey": li["l_partkey"], "l_quantity": li["l_quantity"]}
    plan = _plan(corr_op="=", agg="avg", outer_op="<", outer_key=["l_partkey"], inner_key=["l_partkey"],
                 agg_col="l_quantity", outer_cmp_col="l_quantity", lhs_mult=5, rhs_mult=1,
                 outer_preds=[{"col": "p_brand", "op": "=", "lit": brand_code(2, 3)},
                              {"col": "p_container", "op": "=", "lit": container_code("MED", "BOX")}])
    return {"R": R, "S": S}, plan


def q4(T):
    """TPC-H Q4: orders in [1993-07-01, 1993-10-01) with EXISTS a
    lineitem of the order whose l_commitdate < l_receiptdate (semi-join)."""
    o = T["orders"]
    li = T["lineitem"]
    R = {"o_orderkey": o["o_orderkey"], "o_orderdate": o["o_orderdate"], "o_orderpriority": o["o_orderpriority"]}
    S = {"l_orderkey": li["l_orderkey"], "l_commitdate": li["l_commitdate"], "l_receiptdate": li["l_receiptdate"]}
    plan = _plan(corr_op="=", agg="exists", outer_key=["o_orderkey"], inner_key=["l_orderkey"],
                 outer_preds=[{"col": "o_orderdate", "op": ">=", "lit": D_1993_07_01},
                              {"col": "o_orderdate", "op": "<", "lit": D_1993_10_01}],
                 inner_preds=[{"col": "l_commitdate", "op": "<", "rhs": "l_receiptdate"}])
    return {"R": R, "S": S}, plan


def q20(T):
    """TPC-H Q20's correlated block: partsupp of 'forest%' parts with
    ps_availqty > 0.5 * SUM(l_quantity) of lineitems with the same
    (partkey, suppkey) shipped in 1994 -> 200*ps_availqty > sum(l_quantity
    in cents) (composite '=' key, R9; multipliers R7).  The outer
    supplier/nation IN-list is harness post-processing."""
    ps = T["partsupp"]
    part = T["part"]
    li = T["lineitem"]
    R = {"ps_partkey": ps["ps_partkey"], "ps_suppkey": ps["ps_suppkey"], "ps_availqty": ps["ps_availqty"],
         "p_forest": (part["p_name1"][ps["ps_partkey"] - 1] == FOREST).astype(np.int32)}
    S = {"l_partkey": li["l_partkey"], "l_suppkey": li["l_suppkey"], "l_quantity": li["l_quantity"],
         "l_shipdate": li["l_shipdate"]}
    plan = _plan(corr_op="=", agg="sum", outer_op=">", outer_key=["ps_partkey", "ps_suppkey"],
                 inner_key=["l_partkey", "l_suppkey"], agg_col="l_quantity", outer_cmp_col="ps_availqty",
                 lhs_mult=200, rhs_mult=1,
                 outer_preds=[{"col": "p_forest", "op": "=", "lit": 1}],
                 inner_preds=[{"col": "l_shipdate", "op": ">=", "lit": D_1994_01_01},
                              {"col": "l_shipdate", "op": "<", "lit": D_1995_01_01}])
    return {"R": R, "S": S}, plan


def q20_levels(T):
    """The full three-level TPC-H Q20 (subquery in subquery, Fig. 6):

      level 2  p_partkey IN (part WHERE p_name LIKE 'forest%')   uncorrelated
               -> a host flag column (R10), as in q20
      level 1  partsupp rows with ps_availqty > 0.5*SUM(l_quantity) of their
               (partkey, suppkey) lineitems shipped in 1994  -> q20's plan
      level 0  supplier rows of nation CANADA with s_suppkey IN (level 1's
               ps_suppkey) -- an IN over the level-1 result set, evaluated
               as EXISTS(... WHERE ps_suppkey = s_suppkey) (R10b).

    Returns (level1 tables, level1 plan, carry column name in level1's R --
    the partsupp column level 0's subquery reads --, level0 R table,
    level0 plan whose S is {"ps_suppkey": <level-1 survivors' ps_suppkey>})."""
    tables1, plan1 = q20(T)
    canada = [n for n, _ in NATIONS].index("CANADA")
    R0 = {"s_suppkey": T["supplier"]["s_suppkey"],
          "s_canada": (T["supplier"]["s_nationkey"] == canada).astype(np.int32)}
    plan0 = _plan(corr_op="=", agg="exists", outer_key=["s_suppkey"], inner_key=["ps_suppkey"],
                  outer_preds=[{"col": "s_canada", "op": "=", "lit": 1}])
    return tables1, plan1, "ps_suppkey", R0, plan0


QUERIES = {"q2": q2, "q5": q5, "q17": q17, "q4": q4, "q20": q20}
# BASELINE.json configs[2] = C3 (SF1 Q2, Q17), configs[3] = C4 (SF10 Q4, Q20)
CONFIGS = {"C3": (1.0, ("q2", "q17"), 3), "C4": (10.0, ("q4", "q20"), 5)}


def flattened(query, sf, seed):
    return QUERIES[query](base_tables(sf, seed))
