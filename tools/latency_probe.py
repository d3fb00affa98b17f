"""Host-side latency breakdown of small queries (VERDICT r1 'next' item 4):
wall time of each public call (build_index, exec, result_to_host) and of the
whole query, p50 over many runs, for C1, SF1 Q2 and C2 '=' MIN.

usage: python tools/latency_probe.py [--runs 200]"""
import argparse
import json
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--runs", type=int, default=200)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    from datagen import make_plan, query1, tpch
    from paper_conf_icde_floratosxwgylz21_b200 import Engine
    from tests.gpu_helpers import load
    eng = Engine(0, arena_bytes=2 << 30)
    cases = [("C1 = min", query1.config("C1"), make_plan("=", "min", "="), True),
             ("C1 > min", query1.config("C1"), make_plan(">", "min", "="), False)]
    q2, p2 = tpch.flattened("q2", 1.0, 3)
    cases.append(("SF1 Q2", q2, p2, True))
    c2 = query1.config("C2")
    cases += [("C2 = min", c2, make_plan("=", "min", "="), True), ("C2 = count", c2, make_plan("=", "count", "="), True)]
    out = []
    for name, t, plan, use_index in cases:
        m0 = eng.mark()
        R, S = load(eng, t)
        n_r = len(next(iter(t["R"].values())))
        bufs = {k: torch.empty(max(1, n_r), dtype=d, pin_memory=True).numpy()
                for k, d in (("row", torch.int64), ("value", torch.int64), ("valid", torch.uint8),
                             ("passed", torch.uint8), ("sum", torch.int64), ("cnt", torch.int64))}
        tb, te, th, tt, tp, tpp = [], [], [], [], [], []
        for i in range(a.runs + 10):
            m = eng.mark()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            idx = eng.index_for_plan(plan, S) if use_index else -1
            t1 = time.perf_counter()
            res = eng.exec(plan, R, S, index=idx)
            t2 = time.perf_counter()
            eng.result_to_numpy(res, out=bufs)
            t3 = time.perf_counter()
            eng.release(m)
            # the same query with the plan marshalled once (Engine.prepare)
            m = eng.mark()
            idx = eng.index_for_plan(plan, S) if use_index else -1
            prep = eng.prepare(plan, R, S, index=idx)
            torch.cuda.synchronize()
            eng.release(m)
            m = eng.mark()
            torch.cuda.synchronize()
            u0 = time.perf_counter()
            if use_index:
                eng.index_for_plan(plan, S)   # same index id as at prepare time (same arena state)
            res = eng.exec(prep)
            eng.result_to_numpy(res, out=bufs)
            u1 = time.perf_counter()
            eng.release(m)
            if i >= 10:
                tb.append((t1 - t0) * 1e3)
                te.append((t2 - t1) * 1e3)
                th.append((t3 - t2) * 1e3)
                tt.append((t3 - t0) * 1e3)
                tpp.append((u1 - u0) * 1e3)
        eng.set_profiling(True)
        m = eng.mark()
        idx = eng.index_for_plan(plan, S) if use_index else -1
        eng.exec(plan, R, S, index=idx)
        prof = eng.last_profile()
        eng.release(m)
        eng.set_profiling(False)
        launches0 = eng.launch_count()
        m = eng.mark()
        idx = eng.index_for_plan(plan, S) if use_index else -1
        res = eng.exec(plan, R, S, index=idx)
        eng.result_to_numpy(res, out=bufs)
        eng.release(m)
        rec = {"case": name, "p50_ms": statistics.median(tt), "p90_ms": sorted(tt)[int(0.9 * len(tt))],
               "build_index_p50_ms": statistics.median(tb), "exec_p50_ms": statistics.median(te),
               "to_host_p50_ms": statistics.median(th),
               "prepared_p50_ms": statistics.median(tpp), "launches": eng.launch_count() - launches0,
               "device_stages_ms": {k: v for k, v in prof.items() if v == v}, "survivors": int(res.n_rows)}
        print(json.dumps(rec), flush=True)
        out.append(rec)
        eng.release(m0)
    if a.out:
        with open(a.out, "a") as f:
            for r in out:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
