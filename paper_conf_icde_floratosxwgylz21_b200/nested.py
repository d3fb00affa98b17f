"""Multi-level nested queries on the engine (Fig. 6:
"subquery in a subquery" -- the generated drive program evaluates the
innermost correlated block first; its result vector feeds the block above).

A level is one template plan.  `exec_levels` runs the levels innermost first;
the survivors of level i project one of its R columns (gathered on the
device, nestgpu_gather_column) into the subquery table S of level i+1.
Argument marshalling only -- every step runs in libnestgpu's kernels.
"""


def exec_levels(eng, levels, emit_all=False):
    """levels: innermost first, each a dict
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
