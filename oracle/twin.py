"""Pure-Python twin of the C oracle for tiny inputs (<= ~1e4 pairs).

TEST INFRASTRUCTURE ONLY.  Same semantics as nestgpu_oracle.c -- PAPER.md
Fig. 2 nested loop with the SQL readings R1-R8 of DESIGN.md --
written independently with Python integers (exact, no width limits) and
``fractions.Fraction`` for AVG, so a slip in the C code's integer handling
shows up as a disagreement (tests/test_oracle_pins.py::test_twin_agrees).
"""
from fractions import Fraction

_CMP = {
    "=": lambda x, y: x == y, "!=": lambda x, y: x != y,
    "<": lambda x, y: x < y, "<=": lambda x, y: x <= y,
    ">": lambda x, y: x > y, ">=": lambda x, y: x >= y,
}


def _val(tables, t, c, i):
    m = (tables.get(t + "_valid") or {}).get(c)
    if m is not None and not m[i]:
        return None
    return int(tables[t][c][i])


def _pred(tables, t, p, i):
    x = _val(tables, t, p["col"], i)
    y = _val(tables, t, p["rhs"], i) if p.get("rhs") else int(p["lit"])
    return x is not None and y is not None and _CMP[p["op"]](x, y)


def _round_half_away(q):
    # q is a Fraction; |q| rounded with ties away from zero.
    mag = abs(q)
    r = int(mag + Fraction(1, 2))  # floor(mag + 1/2)
    return r if q >= 0 else -r


def evaluate(tables, plan):
    nR = len(next(iter(tables["R"].values())))
    nS = len(next(iter(tables["S"].values())))
    out = []
    for r in range(nR):
        if not all(_pred(tables, "R", p, r) for p in plan["outer_preds"]):
            out.append(dict(row=r, in_rp=0, passed=0, valid=0, value=0, sum=0, cnt=0))
            continue
        vals = []
        n = 0
        for s in range(nS):
            if not all(_pred(tables, "S", p, s) for p in plan["inner_preds"]):
                continue
            ok = True
            for k, (oc, ic) in enumerate(zip(plan["outer_key"], plan["inner_key"])):
                op = plan["corr_op"] if len(plan["outer_key"]) == 1 else "="
                x = _val(tables, "R", oc, r)
                y = _val(tables, "S", ic, s)
                if x is None or y is None or not _CMP[op](x, y):
                    ok = False
                    break
            if not ok:
                continue
            n += 1
            if plan["agg_col"]:
                v = _val(tables, "S", plan["agg_col"], s)
                if v is not None:
                    vals.append(v)
        agg = plan["agg"]
        valid, value, sm, cnt = 1, 0, 0, n
        if agg == "min":
            valid = bool(vals); value = min(vals) if vals else 0
        elif agg == "max":
            valid = bool(vals); value = max(vals) if vals else 0
        elif agg == "sum":
            valid = bool(vals); value = sum(vals); sm = value
        elif agg == "count":
            value = n
        elif agg == "avg":
            valid = bool(vals); sm = sum(vals); cnt = len(vals)
            value = _round_half_away(Fraction(sm * 10 ** 6, cnt)) if vals else 0
        elif agg == "exists":
            value = int(n > 0)
        elif agg == "not_exists":
            value = int(n == 0)
        if agg in ("exists", "not_exists"):
            passed = value
        else:
            x = _val(tables, "R", plan["outer_cmp_col"], r)
            a, b = plan["lhs_mult"], plan["rhs_mult"]
            if not valid or x is None:
                passed = 0
            elif agg == "avg":
                passed = int(_CMP[plan["outer_op"]](a * x, b * Fraction(sm, cnt)))
            else:
                passed = int(_CMP[plan["outer_op"]](a * x, b * value))
        if not valid:
            value = 0
        out.append(dict(row=r, in_rp=1, passed=passed, valid=int(valid),
                        value=value, sum=sm, cnt=cnt))
    return out
