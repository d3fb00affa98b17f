"""Closed-form "unnested" CPU checker of the correlated aggregate.

TEST INFRASTRUCTURE ONLY (like the rest of oracle/): used by tests/ to pin the
oracle and to check full-size GPU results on every row, and timed by
bench.py's cpu_baseline leg as the second CPU reference point SURVEY.md
§8(d) names ("full-size closed-form prefix checker").  It is NOT the oracle
(nestgpu_oracle.c is the plain Fig. 2 nested loop) and shares no
code with it or with the CUDA path.

Textbook reduction of a range-correlated aggregate (the unnesting of
P:45-49 generalised to every operator): sort S' by key, prefix / suffix
scans (np.minimum.accumulate, np.cumsum), np.searchsorted per outer key.
Valid for '<', '<=', '>', '>='.  For '!=' it uses total-minus-group
(SUM/COUNT/AVG/EXISTS) and the two best distinct key groups (MIN/MAX).  For
'=' it uses per-key groups (np.unique).  NULL-free integer inputs only.
"""
from fractions import Fraction

import numpy as np


def round_half_away(q):
    mag = abs(q)
    r = int(mag + Fraction(1, 2))
    return r if q >= 0 else -r



def _finish(agg, cnt, s_sum, s_min, s_max):
    """-> (valid, value) per row from per-row aggregates over the qualifying set."""
    cnt = np.asarray(cnt, np.int64)
    if agg == "count":
        return np.ones_like(cnt, dtype=bool), cnt
    if agg == "exists":
        return np.ones_like(cnt, dtype=bool), (cnt > 0).astype(np.int64)
    if agg == "not_exists":
        return np.ones_like(cnt, dtype=bool), (cnt == 0).astype(np.int64)
    valid = cnt > 0
    if agg == "min":
        v = s_min
    elif agg == "max":
        v = s_max
    elif agg == "sum":
        v = s_sum
    else:  # avg: exact rounding via Fraction (independent of the oracle's int128)
        v = np.array([round_half_away(Fraction(int(s) * 10 ** 6, int(c))) if c else 0
                      for s, c in zip(s_sum, cnt)], dtype=np.int64)
    return valid, np.where(valid, v, 0).astype(np.int64)


def closed_form(rkey, skey, sval, corr_op, agg):
    """Per-outer-key aggregate over {s : rkey OP skey} for NULL-free int inputs.

    Returns (valid, value, cnt, sum).  cnt = qualifying rows (nn for AVG)."""
    rkey = np.asarray(rkey, np.int64)
    order = np.argsort(skey, kind="stable")
    K = np.asarray(skey, np.int64)[order]
    V = np.asarray(sval, np.int64)[order]
    N = len(K)
    big, small = np.iinfo(np.int64).max, np.iinfo(np.int64).min
    pmin = np.concatenate([[big], np.minimum.accumulate(V)]) if N else np.array([big])
    pmax = np.concatenate([[small], np.maximum.accumulate(V)]) if N else np.array([small])
    psum = np.concatenate([[0], np.cumsum(V)])
    smin = np.concatenate([np.minimum.accumulate(V[::-1])[::-1], [big]]) if N else np.array([big])
    smax = np.concatenate([np.maximum.accumulate(V[::-1])[::-1], [small]]) if N else np.array([small])
    # binary search of every outer key (needles searched in sorted order and
    # scattered back: the same result, without a cache miss per probe)
    ro = np.argsort(rkey, kind="stable")
    rs = rkey[ro]
    lb = np.empty(len(rkey), np.int64)
    ub = np.empty(len(rkey), np.int64)
    lb[ro] = np.searchsorted(K, rs, side="left")
    ub[ro] = np.searchsorted(K, rs, side="right")
    if corr_op in (">", ">="):       # s.key < r.key  /  s.key <= r.key  -> prefix [0, p)
        p = lb if corr_op == ">" else ub
        cnt, s_sum, s_min, s_max = p, psum[p], pmin[p], pmax[p]
    elif corr_op in ("<", "<="):     # s.key > r.key  /  s.key >= r.key  -> suffix [p, N)
        p = ub if corr_op == "<" else lb
        cnt, s_sum, s_min, s_max = N - p, psum[N] - psum[p], smin[p], smax[p]
    elif corr_op == "=":
        cnt = ub - lb
        s_sum = psum[ub] - psum[lb]
        uk, first = np.unique(K, return_index=True)
        gmin = np.minimum.reduceat(V, first) if N else np.array([], np.int64)
        gmax = np.maximum.reduceat(V, first) if N else np.array([], np.int64)
        gi = np.searchsorted(uk, rkey)
        hit = (gi < len(uk)) & (uk[np.minimum(gi, max(len(uk) - 1, 0))] == rkey) if len(uk) else np.zeros(len(rkey), bool)
        s_min = np.where(hit, gmin[np.minimum(gi, max(len(uk) - 1, 0))] if len(uk) else big, big)
        s_max = np.where(hit, gmax[np.minimum(gi, max(len(uk) - 1, 0))] if len(uk) else small, small)
    elif corr_op == "!=":
        # total minus the r.key group
        cnt = N - (ub - lb)
        s_sum = psum[N] - (psum[ub] - psum[lb])
        uk, first = np.unique(K, return_index=True)
        if len(uk):
            gmin = np.minimum.reduceat(V, first)
            gmax = np.maximum.reduceat(V, first)
        else:
            gmin = gmax = np.array([], np.int64)

        def best_two(g, pick):
            # the two groups with the best extreme value (distinct keys)
            if len(g) == 0:
                return None, None
            o = np.argsort(g if pick == "min" else -g, kind="stable")
            return o[0], (o[1] if len(o) > 1 else None)

        s_min = np.full(len(rkey), big, np.int64)
        s_max = np.full(len(rkey), small, np.int64)
        for g, out, pick in ((gmin, s_min, "min"), (gmax, s_max, "max")):
            b1, b2 = best_two(g, pick)
            if b1 is None:
                continue
            use_second = rkey == uk[b1]
            out[:] = g[b1]
            if b2 is None:
                out[use_second] = big if pick == "min" else small
            else:
                out[use_second] = g[b2]
    else:
        raise ValueError(corr_op)
    valid, value = _finish(agg, cnt, s_sum, s_min, s_max)
    return valid, value, np.asarray(cnt, np.int64), np.asarray(s_sum, np.int64)


_CMP = {"=": lambda a, b: a == b, "!=": lambda a, b: a != b, "<": lambda a, b: a < b,
        "<=": lambda a, b: a <= b, ">": lambda a, b: a > b, ">=": lambda a, b: a >= b}


def outer_passed(x, valid, value, cnt, s_sum, agg, outer_op, lhs_mult=1, rhs_mult=1):
    """The outer comparison of the template (Selection on Res) per R
    row, from the closed-form aggregate: a*x OP b*v for MIN/MAX/SUM/COUNT,
    a*x*nn OP b*sum for AVG (exact, reading R6), the boolean for
    [NOT] EXISTS; NULL aggregates (valid == 0) never pass (reading R1).
    Exact: int64 when the operands provably fit, Python ints otherwise."""
    if agg in ("exists", "not_exists"):
        return np.asarray(value, np.int64) != 0
    x = np.asarray(x, np.int64)
    a, b = int(lhs_mult), int(rhs_mult)
    if agg == "avg":
        lhs = [a * int(xi) * int(c) for xi, c in zip(x, cnt)]
        rhs = [b * int(s) for s in s_sum]
        res = np.array([_CMP[outer_op](u, w) for u, w in zip(lhs, rhs)], bool)
    else:
        v = np.asarray(value, np.int64)
        big = max(int(np.abs(x).max(initial=0)) * a, int(np.abs(v).max(initial=0)) * b)
        if big < (1 << 62):
            res = _CMP[outer_op](x * a, v * b)
        else:
            res = np.array([_CMP[outer_op](a * int(xi), b * int(vi)) for xi, vi in zip(x, v)], bool)
    return np.asarray(valid, bool) & res
