#!/usr/bin/env python
"""Ablations of the paper's design claims on B200 (SURVEY.md §8(d)
"Ablations": context reported beside the configs, not targets).

  index      P:315 / P:673 (§III-D "Indexing", Query 7): the '=' plans with
             the sorted correlated-column index (build INCLUDED, as the paper
             includes it) vs the index-less tiled nested loop.
  vectorize  P:147 / P:317 (§III-D "Vectorization", Fig. 4's drive loop):
             C1 evaluated by ONE vectorised exec vs the unvectorised drive
             program -- one exec per outer tuple (an outer predicate on a
             row-id column selects tuple i), i.e. the per-iteration kernel
             launches and synchronisation the paper's Eq. (1) constant C
             charges per iteration.
  pool       P:147 / P:233-237 (§III-C memory pools): the per-tuple drive
             program with the arena pool vs cudaMalloc/cudaFree per scratch
             allocation (nestgpu_set_option(NESTGPU_OPT_MALLOC_SCRATCH)).

Every variant's results are checked equal to the vectorised run (the same
multiset), so an ablation can never trade correctness for time.  Prints one
JSON object; `--out` appends it to a file (profiles/ keeps the round's).
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def cuda_ms(eng, fn, reps=5):
    import torch
    s = eng.stream
    out = None
    times = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(s)
        out = fn()
        b.record(s)
        torch.cuda.synchronize()
        times.append(a.elapsed_time(b))
    return float(np.median(times)), out


def index_ablation(eng, tables, plans, tag):
    from tests.gpu_helpers import load
    rows = []
    m = eng.mark()
    try:
        R, S = load(eng, tables)
        for plan in plans:
            # timed: index build + exec (device result; the D2H is the same
            # for both variants and is left out)
            def with_index():
                return eng.exec(plan, R, S, index=eng.index_for_plan(plan, S))

            def without_index():
                return eng.exec(plan, R, S, index=-1)

            mk = eng.mark()
            t_idx, _ = cuda_ms(eng, with_index)
            a = eng.result_to_numpy(with_index())
            eng.release(mk)
            t_bnl, _ = cuda_ms(eng, without_index, reps=3)
            b = eng.result_to_numpy(without_index())
            assert np.array_equal(a["row"], b["row"]) and np.array_equal(a["value"], b["value"])
            rows.append({"workload": tag, "plan": "%s %s" % (plan["corr_op"], plan["agg"]),
                         "index_incl_build_ms": round(t_idx, 3), "nested_loop_ms": round(t_bnl, 3),
                         "speedup": round(t_bnl / t_idx, 2), "survivors": int(len(a["row"]))})
    finally:
        eng.release(m)
    return rows


def per_tuple_ablation(eng, tables, plan, mode, malloc_scratch):
    """One exec per outer tuple (Fig. 4's loop without vectorisation)."""
    from paper_conf_icde_floratosxwgylz21_b200.binding import OPT_MALLOC_SCRATCH
    import torch
    n = len(tables["R"]["col1"])
    t = {"R": dict(tables["R"], rid=np.arange(n, dtype=np.int32)), "S": tables["S"]}
    m = eng.mark()
    try:
        R = eng.load_table(t["R"])
        S = eng.load_table(t["S"])
        idx = eng.index_for_plan(plan, S) if mode == "index" else -1
        vec = eng.result_to_numpy(eng.exec(plan, R, S, index=idx))
        eng.set_option(OPT_MALLOC_SCRATCH, 1 if malloc_scratch else 0)
        rows, vals = [], []
        launches0 = eng.launch_count()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for i in range(n):
            p = dict(plan, outer_preds=[{"col": "rid", "op": "=", "lit": i}])
            r = eng.exec(p, R, S, index=idx)
            if r.n_rows:
                o = eng.result_to_numpy(r)
                rows.append(int(o["row"][0]))
                vals.append(int(o["value"][0]))
        torch.cuda.synchronize()
        wall = (time.perf_counter() - t0) * 1e3
        launches = eng.launch_count() - launches0
        eng.set_option(OPT_MALLOC_SCRATCH, 0)
        assert rows == vec["row"].tolist() and vals == vec["value"].tolist(), "per-tuple result differs"
        vt, _ = cuda_ms(eng, lambda: eng.result_to_numpy(eng.exec(plan, R, S, index=idx)))
        return {"tuples": n, "per_tuple_ms": round(wall, 2), "per_tuple_us_each": round(wall * 1e3 / n, 2),
                "kernel_launches": launches, "vectorised_ms": round(vt, 3),
                "vectorised_speedup": round(wall / vt, 1)}
    finally:
        eng.set_option(OPT_MALLOC_SCRATCH, 0)
        eng.release(m)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--skip-tpch", action="store_true")
    args = ap.parse_args()
    from datagen import make_plan, query1, tpch
    from paper_conf_icde_floratosxwgylz21_b200 import Engine
    eng = Engine(0, arena_bytes=8 << 30)
    out = {"tool": "ablations", "gpu": None}
    import torch
    out["gpu"] = torch.cuda.get_device_name(0)

    # index vs nested loop ('=' plans; index build included)
    c2 = query1.config("C2")
    rows = index_ablation(eng, c2, [make_plan("=", a, "=") for a in ("min", "count")]
                          + [make_plan("=", "exists", "=")], "C2 (1M x 1M)")
    if not args.skip_tpch:
        for q in ("q2", "q17"):
            tabs, plan = tpch.flattened(q, 1.0, 3)
            rows += index_ablation(eng, tabs, [plan], "TPC-H-shaped SF1 %s" % q.upper())
    out["index_vs_nested_loop"] = rows

    # vectorised vs per-tuple drive program, pool vs cudaMalloc (C1)
    c1 = query1.config("C1")
    out["vectorise_and_pool"] = []
    for mode, op in (("index", "="), ("bnl", ">")):
        plan = make_plan(op, "min", "=")
        pool = per_tuple_ablation(eng, c1, plan, mode, malloc_scratch=False)
        mal = per_tuple_ablation(eng, c1, plan, mode, malloc_scratch=True)
        out["vectorise_and_pool"].append({
            "workload": "C1 (1000 x 1000)", "plan": "%s min (%s)" % (op, mode),
            "vectorised_ms": pool["vectorised_ms"],
            "per_tuple_pool_ms": pool["per_tuple_ms"], "per_tuple_malloc_ms": mal["per_tuple_ms"],
            "per_tuple_us_each_pool": pool["per_tuple_us_each"], "per_tuple_us_each_malloc": mal["per_tuple_us_each"],
            "launches_per_tuple": round(pool["kernel_launches"] / pool["tuples"], 2),
            "vectorisation_speedup": pool["vectorised_speedup"],
            "pool_speedup_per_tuple": round(mal["per_tuple_ms"] / pool["per_tuple_ms"], 2)})
    eng.close()
    line = json.dumps(out)
    print(line)
    if args.out:
        with open(args.out, "a") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
