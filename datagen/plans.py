"""Plan descriptions for the fixed plan template.

A plan is a plain dict; it names columns by string and operators by their SQL
spelling.  It carries no arithmetic.  The template is the SQL-92 query

    SELECT R.* FROM R
    WHERE <outer_preds(R)>
      AND lhs_mult*R.<outer_cmp_col> <outer_op>
          rhs_mult*(SELECT AGG(S.<agg_col>) FROM S
                    WHERE <inner_preds(S)> AND R.<outer_key> <corr_op> S.<inner_key>)

or, for ``agg in {"exists", "not_exists"}``,

    SELECT R.* FROM R WHERE <outer_preds(R)> AND [NOT] EXISTS (SELECT * FROM S WHERE ...)

which is Query 1 generalised to any correlated operator
 and any aggregate (type-JA), following Fig. 4's drive program
(P:175-183): the correlated outer column (R.col2 there) may differ from the
compared outer column (R.col1).

A composite correlation (``outer_key`` / ``inner_key`` of length 2) means
``R.k1 = S.k1 AND R.k2 = S.k2``; only ``corr_op == "="`` is allowed for it
(reading R9).

Predicates: ``{"col": name, "op": sql_op, "lit": int}`` or
``{"col": name, "op": sql_op, "rhs": other_col}`` (same table).
"""

PLAN_OPS = ("=", "!=", "<", "<=", ">", ">=")
PLAN_AGGS = ("min", "max", "sum", "count", "avg", "exists", "not_exists")


def make_plan(corr_op="=", agg="min", outer_op="=", *, outer_key=("col1",),
              inner_key=("col1",), agg_col="col2", outer_cmp_col="col2",
              outer_preds=(), inner_preds=(), lhs_mult=1, rhs_mult=1):
    if corr_op not in PLAN_OPS or outer_op not in PLAN_OPS:
        raise ValueError("bad operator")
    if agg not in PLAN_AGGS:
        raise ValueError("bad aggregate")
    outer_key = tuple(outer_key)
    inner_key = tuple(inner_key)
    if len(outer_key) != len(inner_key) or len(outer_key) not in (1, 2):
        raise ValueError("key arity")
    return {
        "outer_preds": [dict(p) for p in outer_preds],
        "outer_key": list(outer_key),
        "inner_key": list(inner_key),
        "corr_op": corr_op,
        "inner_preds": [dict(p) for p in inner_preds],
        "agg": agg,
        "agg_col": agg_col if agg not in ("count", "exists", "not_exists") else None,
        "outer_cmp_col": outer_cmp_col if agg not in ("exists", "not_exists") else None,
        "outer_op": outer_op,
        "lhs_mult": int(lhs_mult),
        "rhs_mult": int(rhs_mult),
    }


def plan_columns(plan):
    """(R columns, S columns) referenced by a plan, in first-use order."""
    rc, sc = [], []

    def add(lst, c):
        if c is not None and c not in lst:
            lst.append(c)

    for p in plan["outer_preds"]:
        add(rc, p["col"])
        add(rc, p.get("rhs"))
    for c in plan["outer_key"]:
        add(rc, c)
    add(rc, plan["outer_cmp_col"])
    for p in plan["inner_preds"]:
        add(sc, p["col"])
        add(sc, p.get("rhs"))
    for c in plan["inner_key"]:
        add(sc, c)
    add(sc, plan["agg_col"])
    return rc, sc
