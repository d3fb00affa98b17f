"""Python front-end for the CPU oracle (oracle/nestgpu_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs; never by the product path.
It shares nothing with paper_conf_icde_floratosxwgylz21_b200/ and include/.

Marshalling only: columns are widened to int64 (SQL integers; widening does
not change any comparison, sum or order), NULL masks are passed as bytes,
and the plan dict (datagen.plans) is mapped onto the C struct.  All of the
method's arithmetic is in nestgpu_oracle.c.
"""
import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "nestgpu_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

OPS = {"=": 0, "!=": 1, "<": 2, "<=": 3, ">": 4, ">=": 5}
AGGS = {"min": 0, "max": 1, "sum": 2, "count": 3, "avg": 4, "exists": 5,
        "not_exists": 6}


class OracleOverflow(ArithmeticError):
    pass


def build(force=False):
    """Compile liboracle.so with gcc -O2 -fopenmp (plain C, no CUDA)."""
    if (not force and os.path.exists(_LIB)
            and os.path.getmtime(_LIB) >= os.path.getmtime(_SRC)):
        return _LIB
    tmp = _LIB + ".%d.tmp" % os.getpid()
    subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC",
                           "-std=c11", "-Wall", "-o", tmp, _SRC])
    os.replace(tmp, _LIB)
    return _LIB


class _Col(ctypes.Structure):
    _fields_ = [("v", ctypes.c_void_p), ("valid", ctypes.c_void_p)]


class _Pred(ctypes.Structure):
    _fields_ = [("col", ctypes.c_int32), ("op", ctypes.c_int32),
                ("lit", ctypes.c_int64), ("rhs_col", ctypes.c_int32)]


class _Corr(ctypes.Structure):
    _fields_ = [("outer_col", ctypes.c_int32), ("op", ctypes.c_int32),
                ("inner_col", ctypes.c_int32)]


class _Plan(ctypes.Structure):
    _fields_ = [("nR", ctypes.c_int64), ("nS", ctypes.c_int64),
                ("R", ctypes.c_void_p), ("S", ctypes.c_void_p),
                ("outer_preds", ctypes.c_void_p), ("n_outer", ctypes.c_int32),
                ("corr", ctypes.c_void_p), ("n_corr", ctypes.c_int32),
                ("inner_preds", ctypes.c_void_p), ("n_inner", ctypes.c_int32),
                ("agg", ctypes.c_int32), ("agg_col", ctypes.c_int32),
                ("cmp_col", ctypes.c_int32), ("outer_op", ctypes.c_int32),
                ("a", ctypes.c_int64), ("b", ctypes.c_int64)]


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            lib.oracle_eval.restype = ctypes.c_int
            lib.oracle_eval.argtypes = [ctypes.c_void_p] * 11 + [ctypes.c_int]
            lib.oracle_eval.argtypes[2] = ctypes.c_int64
            lib.oracle_max_threads.restype = ctypes.c_int
            _lib = lib
    return _lib


def max_threads():
    return _load().oracle_max_threads()


def _ptr(a):
    return None if a is None else a.ctypes.data


def _make_plan(tables, plan):
    """Map (tables, plan dict) onto the C oplan (widening to int64).
    Returns (oplan, objects to keep alive, nR)."""
    keep = []

    def table(name):
        cols = tables[name]
        valids = tables.get(name + "_valid", {}) or {}
        names = list(cols)
        arr = (_Col * max(1, len(names)))()
        n = None
        for i, c in enumerate(names):
            v = np.ascontiguousarray(cols[c], dtype=np.int64)
            n = len(v) if n is None else n
            if len(v) != n:
                raise ValueError("ragged table %s" % name)
            keep.append(v)
            arr[i].v = v.ctypes.data
            m = valids.get(c)
            if m is not None:
                m = np.ascontiguousarray(m, dtype=np.uint8)
                keep.append(m)
                arr[i].valid = m.ctypes.data
            else:
                arr[i].valid = None
        keep.append(arr)
        return names, arr, (n or 0)

    rnames, rarr, nR = table("R")
    snames, sarr, nS = table("S")

    def preds(lst, names):
        arr = (_Pred * max(1, len(lst)))()
        for i, p in enumerate(lst):
            arr[i].col = names.index(p["col"])
            arr[i].op = OPS[p["op"]]
            if "rhs" in p and p["rhs"] is not None:
                arr[i].rhs_col = names.index(p["rhs"])
                arr[i].lit = 0
            else:
                arr[i].rhs_col = -1
                arr[i].lit = int(p["lit"])
        keep.append(arr)
        return arr, len(lst)

    op_arr, n_op = preds(plan["outer_preds"], rnames)
    ip_arr, n_ip = preds(plan["inner_preds"], snames)
    corr = (_Corr * 2)()
    keep.append(corr)
    for i, (oc, ic) in enumerate(zip(plan["outer_key"], plan["inner_key"])):
        corr[i].outer_col = rnames.index(oc)
        corr[i].inner_col = snames.index(ic)
        # composite keys are equality on every component (reading R9)
        corr[i].op = OPS[plan["corr_op"]] if len(plan["outer_key"]) == 1 else OPS["="]
    if len(plan["outer_key"]) == 2 and plan["corr_op"] != "=":
        raise ValueError("composite correlation must be '='")

    P = _Plan()
    P.nR, P.nS = nR, nS
    P.R, P.S = ctypes.addressof(rarr), ctypes.addressof(sarr)
    P.outer_preds, P.n_outer = ctypes.addressof(op_arr), n_op
    P.corr, P.n_corr = ctypes.addressof(corr), len(plan["outer_key"])
    P.inner_preds, P.n_inner = ctypes.addressof(ip_arr), n_ip
    P.agg = AGGS[plan["agg"]]
    P.agg_col = snames.index(plan["agg_col"]) if plan["agg_col"] else -1
    P.cmp_col = rnames.index(plan["outer_cmp_col"]) if plan["outer_cmp_col"] else -1
    P.outer_op = OPS[plan["outer_op"]]
    P.a, P.b = plan["lhs_mult"], plan["rhs_mult"]

    return P, keep, nR


def evaluate(tables, plan, rows=None, s_window=None, threads=0):
    """Evaluate ``plan`` over ``tables`` (datagen layout: {"R": {name: arr},
    "S": {...}, optional "R_valid"/"S_valid"}).

    rows     : optional int64 array of R row numbers to evaluate (a sample);
               default all rows in order.
    s_window : optional (lo, hi) int64 arrays, per evaluated row, restricting
               S to rows [lo, hi) -- used to batch many tiny instances.
    Returns a dict of numpy arrays, one entry per evaluated row:
    row, in_rp, passed, valid, value, sum, cnt.
    """
    lib = _load()
    P, keep, nR = _make_plan(tables, plan)

    if rows is None:
        rows_arr = None
        n_eval = nR
    else:
        rows_arr = np.ascontiguousarray(rows, dtype=np.int64)
        n_eval = len(rows_arr)
    lo = hi = None
    if s_window is not None:
        lo = np.ascontiguousarray(s_window[0], dtype=np.int64)
        hi = np.ascontiguousarray(s_window[1], dtype=np.int64)
        assert len(lo) == len(hi) == n_eval
    out = {
        "in_rp": np.zeros(n_eval, np.uint8),
        "passed": np.zeros(n_eval, np.uint8),
        "valid": np.zeros(n_eval, np.uint8),
        "value": np.zeros(n_eval, np.int64),
        "sum": np.zeros(n_eval, np.int64),
        "cnt": np.zeros(n_eval, np.int64),
    }
    st = lib.oracle_eval(ctypes.addressof(P), _ptr(rows_arr), n_eval,
                         _ptr(lo), _ptr(hi),
                         out["in_rp"].ctypes.data, out["passed"].ctypes.data,
                         out["valid"].ctypes.data, out["value"].ctypes.data,
                         out["sum"].ctypes.data, out["cnt"].ctypes.data,
                         int(threads))
    if st == -5:
        raise OracleOverflow("sum exceeds int64")
    if st != 0:
        raise ValueError("oracle rejected plan (%d)" % st)
    out["row"] = (np.arange(nR, dtype=np.int64) if rows_arr is None else rows_arr)
    return out


def collect(tables, plan):
    """Type-J subquery results as the paper's two-level arrays:
    for every R row, the non-NULL values of plan["agg_col"] over the S rows
    that satisfy the inner predicates and the correlation (reading R17).
    Returns {"in_rp", "lens" (level 1), "offsets" (exclusive prefix of lens,
    nR + 1 entries), "values" (level 2, per row in S row order)}.  Marshalling
    only; the arithmetic is oracle_collect in nestgpu_oracle.c."""
    lib = _load()
    if not hasattr(lib, "_collect_ready"):
        lib.oracle_collect.restype = ctypes.c_int
        lib.oracle_collect.argtypes = [ctypes.c_void_p] * 4 + [ctypes.c_int64]
        lib._collect_ready = True
    P, keep, nR = _make_plan(tables, plan)
    in_rp = np.zeros(nR, np.uint8)
    lens = np.zeros(nR, np.int64)
    st = lib.oracle_collect(ctypes.addressof(P), in_rp.ctypes.data, lens.ctypes.data, None, 0)
    if st != 0:
        raise ValueError("oracle rejected plan (%d)" % st)
    total = int(lens.sum())
    vals = np.zeros(max(total, 1), np.int64)
    st = lib.oracle_collect(ctypes.addressof(P), None, lens.ctypes.data, vals.ctypes.data, total)
    if st != 0:
        raise ValueError("oracle collect failed (%d)" % st)
    offsets = np.zeros(nR + 1, np.int64)
    np.cumsum(lens, out=offsets[1:])
    del keep
    return {"in_rp": in_rp, "lens": lens, "offsets": offsets, "values": vals[:total]}


def in_list(tables, plan, x_col):
    """x IN (SELECT S.v FROM S WHERE ... correlated ...) per R row, read off
    the two-level arrays of ``collect`` (the upper-level selection consuming a
    type-J result).  SQL: TRUE iff x is not NULL and some element
    equals it (NULL elements are never materialised, reading R17, and never
    make IN TRUE).  Returns (in_rp, passed) uint8 arrays."""
    c = collect(tables, plan)
    x = np.asarray(tables["R"][x_col], dtype=np.int64)
    xv = (tables.get("R_valid", {}) or {}).get(x_col)
    passed = np.zeros(len(x), np.uint8)
    for r in range(len(x)):
        if not c["in_rp"][r] or (xv is not None and not xv[r]):
            continue
        lst = c["values"][c["offsets"][r]:c["offsets"][r + 1]]
        passed[r] = 1 if any(int(v) == int(x[r]) for v in lst) else 0
    return c["in_rp"], passed


def survivors(res):
    """(row ids, values) of the result multiset (rows whose predicate held)."""
    m = res["passed"].astype(bool)
    return res["row"][m], res["value"][m]
