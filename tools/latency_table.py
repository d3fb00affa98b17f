"""Query latency of every BASELINE.json config on one GPU (SURVEY.md §8(d)
record schema): C1 (both plans), C2 (the 12-plan sweep), C3a SF1 Q2, C3b SF1
Q17, C4a SF10 Q4, C4b SF10 Q20, C5 16M '>' MIN.

Latency = build_index (inner filter + sort; '=' plans) + exec_correlated +
result_to_host (into pinned host buffers allocated once and reused), wall
clock from a synchronised start until the survivors are in host memory,
columns resident (the paper includes index build, and
excludes disk I/O).  The strategy is the paper's: the index for '='
correlations, the nested loop otherwise.  Per-stage device
times come from one extra profiled run (nestgpu_last_profile).

usage: python tools/latency_table.py [--out profiles/r01_latency.jsonl] [--skip-c5]
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

ALU_PAIRS_PER_CLK = {"min": 32.0, "max": 32.0, "count": 64.0, "sum": 32.0, "avg": 32.0}


def ideal_stages(tabs, plan, st, use_index, survivors, hbm_gbps, alu_ms):
    """Ideal time (ms) of each stage from the ALGORITHMIC work (SURVEY.md
    §8(d)): HBM stages move their bytes at the measured copy bandwidth, the
    nested loop runs at its integer-pipe bound.  Bytes per stage:
      S' filter  n_S x (inner predicate + key + payload column widths) read
                 + |S'| x (key + payload) written
      sort       one read + one write of |S'| x (key + payload) (lower bound;
                 none for a key-ordered column, which the engine does not sort)
      R' filter  n_R x (outer predicate + key column widths) read
                 + |R'| x (4-byte id + key) written
      probe      |R'| x key read + sum_k x payload read + |R'| x 16 B partials
      finalize   |R'| x (16 B partials + id + compared column) read
                 + survivors x 18 B written"""
    R, S = tabs["R"], tabs["S"]

    def w(t, c):
        return t[c].dtype.itemsize

    kb = 4 if (len(plan["inner_key"]) == 1 and w(S, plan["inner_key"][0]) == 4) else 8
    vb = w(S, plan["agg_col"]) if plan.get("agg_col") else 0
    n_r, n_s = len(next(iter(R.values()))), len(next(iter(S.values())))
    in_cols = {p["col"] for p in plan["inner_preds"]} | {p["rhs"] for p in plan["inner_preds"] if p.get("rhs")}
    in_w = sum(w(S, c) for c in in_cols | set(plan["inner_key"]) | ({plan["agg_col"]} if vb else set()))
    out_cols = {p["col"] for p in plan["outer_preds"]} | {p["rhs"] for p in plan["outer_preds"] if p.get("rhs")}
    out_w = sum(w(R, c) for c in out_cols | set(plan["outer_key"]))
    xw = w(R, plan["outer_cmp_col"]) if plan.get("outer_cmp_col") else 0
    b = {"inner_filter": n_s * in_w + st["n_sp"] * (kb + vb),
         "outer_filter": n_r * out_w + st["n_rp"] * (4 + kb),
         "finalize": st["n_rp"] * (16 + 4 + xw) + survivors * 18}
    if use_index and st["sort_passes"] > 0:   # key-ordered columns need no sort (cost_model.stats)
        b["sort"] = 2 * st["n_sp"] * (kb + vb)
    if use_index:
        b["probe"] = st["n_rp"] * (kb + 16) + st["sum_k"] * vb
    out = {k: v / (hbm_gbps * 1e9) * 1e3 for k, v in b.items()}
    if not use_index:
        out["nested_loop"] = alu_ms
    return out, b


def cases(skip_c5):
    from datagen import make_plan, query1, tpch
    out = []
    c1 = query1.config("C1")
    out += [("C1", c1, make_plan("=", "min", "="), 1), ("C1", c1, make_plan(">", "min", "="), 1)]
    c2 = query1.config("C2")
    out += [("C2", c2, make_plan(op, agg, "="), 2) for op, agg in query1.C2_SWEEP]
    for cfg, q, sf, seed in (("C3a", "q2", 1.0, 3), ("C3b", "q17", 1.0, 3), ("C4a", "q4", 10.0, 5),
                             ("C4b", "q20", 10.0, 5)):
        tabs, plan = tpch.flattened(q, sf, seed)
        out.append(("%s SF%g %s" % (cfg, sf, q.upper()), tabs, plan, seed))
    if not skip_c5:
        out.append(("C5", query1.config("C5"), make_plan(">", "min", "="), 7))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--skip-c5", action="store_true")
    args = ap.parse_args()
    import torch
    from paper_conf_icde_floratosxwgylz21_b200 import Engine
    from tests.gpu_helpers import load
    from tools.cost_model import stats

    eng = Engine(0, arena_bytes=24 << 30)
    props = torch.cuda.get_device_properties(0)
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    sm_mhz = float(peaks.get("sm_max_mhz", 1965))
    from paper_conf_icde_floratosxwgylz21_b200 import nested
    params = eng.cost_calibrate()
    pinned = {}

    def res_buffers(n):
        # pinned host result buffers, allocated once (outside the timed region)
        # and reused -- the copy then runs at PCIe speed (binding result_to_numpy(out=))
        if not pinned or len(pinned["row"]) < n:
            pinned.clear()
            pinned.update({k: torch.empty(n, dtype=dt, pin_memory=True).numpy()
                           for k, dt in (("row", torch.int64), ("value", torch.int64), ("valid", torch.uint8),
                                         ("passed", torch.uint8), ("sum", torch.int64), ("cnt", torch.int64))})
        return pinned

    for name, tabs, plan, seed in cases(args.skip_c5):
        m = eng.mark()
        R, S = load(eng, tabs)
        out = res_buffers(len(next(iter(tabs["R"].values()))))
        use_index = plan["corr_op"] == "="
        reps = args.reps if name != "C5" else 2
        warm = 3 if name != "C5" else 1
        lat = []
        res_n = None
        for r in range(warm + reps):
            mk = eng.mark()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            idx = eng.index_for_plan(plan, S) if use_index else -1
            res = eng.exec(plan, R, S, index=idx)
            host = eng.result_to_numpy(res, out=out)
            t1 = time.perf_counter()
            if r >= warm:
                lat.append(1e3 * (t1 - t0))
            res_n = len(host["row"])
            eng.release(mk)
        eng.set_profiling(True)
        mk = eng.mark()
        idx = eng.index_for_plan(plan, S) if use_index else -1
        eng.exec(plan, R, S, index=idx)
        stages = eng.last_profile()
        ix_prof = None
        eng.release(mk)
        if use_index:   # build_index alone: its inner filter + sort stages
            mk = eng.mark()
            eng.index_for_plan(plan, S)
            ix_prof = eng.last_profile()
            eng.release(mk)
        eng.set_profiling(False)
        # the cost model's choice (§IV): nested.exec_auto
        st = stats(tabs, plan, res_n)
        cin = {k: st[k] for k in ("n_r", "n_s", "n_rp", "n_sp", "n_distinct", "sum_k", "survivors", "key_bytes",
                                  "payload_bytes", "sort_passes", "dedup_passes", "corr_op", "agg", "narrow_keys")}
        alat, strategy = [], None
        for r in range(warm + reps):
            mk = eng.mark()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            res, strategy, _ = nested.exec_auto(eng, plan, R, S, params, cin)
            host = eng.result_to_numpy(res, out=out)
            t1 = time.perf_counter()
            if r >= warm:
                alat.append(1e3 * (t1 - t0))
            assert len(host["row"]) == res_n, (name, strategy)
            eng.release(mk)
        eng.release(m)
        n_r = len(next(iter(tabs["R"].values())))
        n_s = len(next(iter(tabs["S"].values())))
        p50 = float(np.median(lat))
        rec = {"config": name, "plan": "%s %s" % (plan["corr_op"], plan["agg"]), "seed": seed, "world_size": 1,
               "strategy": "index" if use_index else "nested_loop", "n_R": n_r, "n_S": n_s,
               "survivors": res_n, "latency_ms": {"p50": p50, "p90": float(np.percentile(lat, 90)),
                                                  "runs": len(lat)},
               "outer_tuples_per_s": n_r / (p50 / 1e3),
               "stages_ms": {k: round(v, 4) for k, v in stages.items()},
               "gpu": props.name}
        if ix_prof:
            rec["index_build_ms"] = {"inner_filter": round(ix_prof["inner_filter"], 4),
                                     "sort": round(ix_prof["sort"], 4)}
        rec["cost_model_choice"] = {"strategy": strategy, "latency_ms_p50": float(np.median(alat)),
                                    "outer_tuples_per_s": n_r / (float(np.median(alat)) / 1e3)}
        rec.update({"n_Rp": st["n_rp"], "n_Sp": st["n_sp"], "sum_k": st["sum_k"], "sort_passes": st["sort_passes"]})
        if not use_index and plan["agg"] in ALU_PAIRS_PER_CLK and stages.get("subquery", 0) > 0:
            # the nested-loop kernel against its integer-pipe bound
            pairs = st["n_rp"] * st["n_sp"]
            ideal = pairs / (props.multi_processor_count * ALU_PAIRS_PER_CLK[plan["agg"]] * sm_mhz * 1e6) * 1e3
            rec["pairs"] = pairs
            rec["pairs_per_s"] = pairs / (stages["subquery"] / 1e3)
            rec["nested_loop_alu_frac"] = ideal / stages["subquery"]
        hbm = float(peaks.get("hbm_gbs", 6454.6))   # measured copy bandwidth (MEASURED_PEAKS.json)
        alu_ms = None
        if not use_index and plan["agg"] in ALU_PAIRS_PER_CLK:
            alu_ms = st["n_rp"] * st["n_sp"] / (props.multi_processor_count * ALU_PAIRS_PER_CLK[plan["agg"]]
                                                * sm_mhz * 1e6) * 1e3
        if use_index or alu_ms is not None:
            ideal, nbytes = ideal_stages(tabs, plan, st, use_index, res_n, hbm, alu_ms)
            ideal_total = sum(ideal.values())
            dev = stages["total"] + (sum(ix_prof[k] for k in ("inner_filter", "sort") if ix_prof[k] == ix_prof[k])
                                     if ix_prof else 0.0)
            rec["roofline"] = {"ideal_ms": {k: round(v, 5) for k, v in ideal.items()},
                               "algorithmic_bytes": nbytes, "hbm_gbps": hbm,
                               "query_frac": ideal_total / p50, "device_frac": ideal_total / dev if dev > 0 else None}
        print(json.dumps(rec), flush=True)
        if args.out:
            with open(args.out, "a") as f:
                f.write(json.dumps(rec) + "\n")
    eng.close()


if __name__ == "__main__":
    main()
