"""Helpers for the -m gpu parity tests: run a plan through the C ABI and
compare with the oracle element by element."""
import numpy as np

import oracle
from paper_conf_icde_floratosxwgylz21_b200 import Engine


def load(eng, tables, dtypes=None):
    dtypes = dtypes or {}
    R = eng.load_table(tables["R"], tables.get("R_valid"), dtypes.get("R"))
    S = eng.load_table(tables["S"], tables.get("S_valid"), dtypes.get("S"))
    return R, S


def run(eng, tables, plan, mode="bnl", emit_all=True, dtypes=None, row_id_base=0, dedup=False, with_res=False):
    """mode: 'bnl' (index=-1) or 'index' (build the index first)."""
    m = eng.mark()
    try:
        R, S = load(eng, tables, dtypes)
        idx = eng.index_for_plan(plan, S) if mode == "index" else -1
        res = eng.exec(plan, R, S, index=idx, emit_all=emit_all, row_id_base=row_id_base, dedup=dedup)
        out = eng.result_to_numpy(res)
        if with_res:
            out["n_evaluated"] = res.n_evaluated
        return out
    finally:
        eng.release(m)


def assert_parity(gpu, ref, plan, emit_all=True, rows=None, ctx=""):
    """Compare a GPU result with an oracle result.

    emit_all: GPU holds every R' tuple -> compare value / valid / passed (and
    AVG sum / nn) row by row.  Otherwise compare the survivor multisets.
    rows: if the oracle evaluated only a sample of rows, restrict the GPU
    result to those rows (GPU must be emit_all then)."""
    if rows is not None:
        assert emit_all
        sel_in = ref["in_rp"].astype(bool)
        pos = np.minimum(np.searchsorted(gpu["row"], rows), max(len(gpu["row"]) - 1, 0))[sel_in]
        assert np.array_equal(gpu["row"][pos], rows[sel_in]), (ctx, "sampled rows missing")
        for k in ("value", "valid", "passed"):
            g = gpu[k][pos].astype(np.int64)
            e = ref[k][sel_in].astype(np.int64)
            if not np.array_equal(g, e):
                bad = np.nonzero(g != e)[0][:5]
                raise AssertionError("%s field %s mismatch at rows %s: gpu %s oracle %s" % (
                    ctx, k, rows[sel_in][bad], g[bad], e[bad]))
        return
    if emit_all:
        m = ref["in_rp"].astype(bool)
        exp_rows = ref["row"][m]
        assert np.array_equal(gpu["row"], exp_rows), (ctx, "rows", len(gpu["row"]), len(exp_rows))
        for k in ("value", "valid", "passed"):
            g = gpu[k].astype(np.int64)
            e = ref[k][m].astype(np.int64)
            if not np.array_equal(g, e):
                bad = np.nonzero(g != e)[0][:5]
                raise AssertionError("%s field %s mismatch at rows %s: gpu %s oracle %s" % (
                    ctx, k, exp_rows[bad], g[bad], e[bad]))
        if plan["agg"] == "avg":
            ok = ref["valid"][m].astype(bool)
            assert np.array_equal(gpu["sum"][ok], ref["sum"][m][ok]), ctx
            assert np.array_equal(gpu["cnt"][ok], ref["cnt"][m][ok]), ctx
    else:
        rows, vals = oracle.survivors(ref)
        assert np.array_equal(gpu["row"], rows), (ctx, "survivor rows", len(gpu["row"]), len(rows))
        assert np.array_equal(gpu["value"], vals), (ctx, "survivor values")
        assert np.all(gpu["passed"] == 1)


def make_engine(arena_gb=8):
    return Engine(0, arena_bytes=int(arena_gb * (1 << 30)))
