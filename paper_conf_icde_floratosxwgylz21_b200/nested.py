"""Multi-level nested queries and joins with subqueries on the engine
(§III-B: Fig. 5 "Generating code for a subquery in
Join", Fig. 6 "subquery in a subquery", type-J results as two-level arrays).

Every function here is a drive program in the paper's sense:
argument marshalling and the order of engine calls only -- every step runs
in libnestgpu's kernels (filters, sorts, binary searches, range aggregates,
nested loops, collections, gathers, materialisations).
"""


def exec_levels(eng, levels, emit_all=False):
    """Subquery in a subquery (Fig. 6): the generated drive program
    evaluates the innermost correlated block first; its result vector feeds
    the block above.  levels: innermost first, each a dict
         plan   : datagen plan dict
         R      : {name: column id}           (this level's outer table)
         S      : {name: column id}           (level 0 only)
         carry  : name of the R column whose values at the survivors become
                  the next level's S column (all levels but the last)
         as     : name of that S column in the next level's plan
         mode   : "index" or "bnl"
    Returns the last level's nestgpu result (device pointers valid until the
    next exec)."""
    S = levels[0]["S"]
    res = None
    for i, lv in enumerate(levels):
        if i > 0:
            prev = levels[i - 1]
            S = {prev["as"]: eng.gather_column(prev["R"][prev["carry"]], res)}
        idx = eng.index_for_plan(lv["plan"], S) if lv.get("mode", "index") == "index" else -1
        res = eng.exec(lv["plan"], lv["R"], S, index=idx, emit_all=emit_all and i == len(levels) - 1)
    return res


def _equi_pairs(eng, probe_tab, probe_key, build_tab, build_key, build_rid):
    """JOIN(=, build.key, probe.key) as type-J collection: an index on
    build.key carrying build's row-id column, probed once per probe row
    (vectorised).  Returns the collection: owner = probe row,
    values = build row id of each matching pair."""
    from datagen import make_plan
    idx = eng.build_index(build_tab, [build_key], payload=build_rid)
    plan = make_plan("=", "min", "=", outer_key=[probe_key], inner_key=[build_key], agg_col=build_rid,
                     outer_cmp_col=probe_key)
    return eng.exec_collect(plan, probe_tab, build_tab, idx)


def _pairs_to_host(eng, left_ptr, right_ptr, n):
    """(left row id, right row id) host arrays from two device int64 vectors."""
    import numpy as np
    import torch
    if n == 0:
        return np.zeros(0, np.int64), np.zeros(0, np.int64)
    a = eng.arena_view(left_ptr, n * 8).view(torch.int64).cpu().numpy()
    b = eng.arena_view(right_ptr, n * 8).view(torch.int64).cpu().numpy()
    return a, b


def join_subquery_right(eng, L, l_key, l_rid, RT, S, plan, mode="index", key_dtype="int32"):
    """Fig. 5, first case: JOIN LEFT.col1 = SUBQ(RIGHT.col1) --
    the subquery is correlated with RIGHT only, so it runs once per RIGHT
    tuple ("for i < RIGHT.tupleNum: Res[i] = Materialize(...)"), then
    "JOIN(=, LEFT.col1, Res)".

      L, RT, S : {name: column id};  l_key: LEFT's join column;  l_rid: a
                 LEFT row-id column;  plan: the subquery as a template plan
                 over R = RIGHT (its outer_cmp / outer_op are not used).
    Steps: exec (emit_all) -> Res[i] per RIGHT' tuple; Res and the RIGHT row
    ids materialised as columns; the equi-join of LEFT.l_key with Res as a
    type-J collection over an index on LEFT.l_key.
    Returns host arrays (left row ids, right row ids) of the joined pairs."""
    idx = eng.index_for_plan(plan, S) if mode == "index" else -1
    res = eng.exec(plan, RT, S, index=idx, emit_all=True)
    n = res.n_rows
    res_col = eng.column_from_device(res.d_values, n, key_dtype, d_valid=res.d_valid)
    rid_col = eng.column_from_device(res.d_row_ids, n, "int64")
    coll = _equi_pairs(eng, {"res": res_col}, "res", L, l_key, l_rid)
    # owner = position in Res -> the RIGHT row id through rid_col
    right = eng.gather_column(rid_col, (coll.d_owner, coll.n_values))
    right_ptr = eng.column_info(right)["d_values"]
    return _pairs_to_host(eng, coll.d_values, right_ptr, coll.n_values)


def join_subquery_both(eng, L, RT, S, join_on, l_rid, sub_plan, mode="index"):
    """Fig. 5, second case: JOIN LEFT.col1 = SUBQ(LEFT.col2,
    RIGHT.col1) -- correlated with both tables, so the paper iterates over
    the Cartesian product.  The paper's optimisation for a natural join with
    AND-ed predicates ("first joining two tables with the predicates
    without correlated subqueries, and then performing a selection over the
    result table") is applied: join on `join_on` = (LEFT col, RIGHT col)
    first, gather the columns the subquery needs into the join table J, then
    run the correlated selection over J.

      sub_plan : template plan over R = J whose columns are named
                 "l.<col>" / "r.<col>" (e.g. outer_key ["l.col2", "r.col1"]
                 with a composite '=' correlation, outer_cmp_col "l.col1").
    Returns host arrays (left row ids, right row ids) of the surviving pairs."""
    lcol, rcol = join_on
    coll = _equi_pairs(eng, RT, rcol, L, lcol, l_rid)
    m = coll.n_values
    need = set(sub_plan["outer_key"]) | {sub_plan.get("outer_cmp_col")} | {p["col"] for p in sub_plan["outer_preds"]}
    J = {}
    for name in sorted(x for x in need if x):
        side, col = name.split(".", 1)
        if side == "l":
            J[name] = eng.gather_column(L[col], (coll.d_values, m))
        else:
            J[name] = eng.gather_column(RT[col], (coll.d_owner, m))
    lid = eng.column_from_device(coll.d_values, m, "int64")
    rid = eng.column_from_device(coll.d_owner, m, "int64")
    idx = eng.index_for_plan(sub_plan, S) if mode == "index" else -1
    res = eng.exec(sub_plan, J, S, index=idx)
    a = eng.gather_column(lid, res)
    b = eng.gather_column(rid, res)
    return _pairs_to_host(eng, eng.column_info(a)["d_values"], eng.column_info(b)["d_values"], res.n_rows)


def exec_auto(eng, plan, R, S, params, stats, emit_all=False, row_id_base=0):
    """Run a plan with the strategy the cost model predicts fastest (P:75,
    §IV: the model "guide[s] subquery processing by selecting the most
    effective execution path").  params: Engine.cost_calibrate(); stats: the
    plan's cardinalities (nestgpu_cost_input fields, known in advance as in
    the paper's evaluation).  Returns (result, strategy, predicted)."""
    from .binding import cost_estimate
    est = cost_estimate(params, **stats)
    strategy = est["best"]
    idx = eng.index_for_plan(plan, S) if strategy.startswith("index") else -1
    res = eng.exec(plan, R, S, index=idx, emit_all=emit_all, row_id_base=row_id_base,
                   dedup=strategy.endswith("cached"))
    return res, strategy, est
